"""Start/end spread of tc_seg CTAs (TCSEG_TIMING + TCSEG_TIMING_ALL build): reads the kernel's
printf lines from stdin and prints, per launch (CTAs grouped by start-time gaps > 100 us), the
quantiles of CTA start and end times relative to the launch's first CTA, and of CTA durations.
Usage: python tools/tcseg_plain_timing.py | python tools/tcseg_waves.py"""
import sys

rows = []
for line in sys.stdin:
    if line.startswith("tcsegall"):
        f = line.split()
        rows.append((int(f[1]), int(f[2]), int(f[3]), int(f[4]), int(f[5])))
rows.sort(key=lambda r: r[3])
groups, cur = [], []
for r in rows:
    if cur and r[3] - cur[-1][3] > 100_000:
        groups.append(cur)
        cur = []
    cur.append(r)
if cur:
    groups.append(cur)


def q(xs, p):
    xs = sorted(xs)
    return xs[min(len(xs) - 1, int(p * len(xs)))]


for g in groups:
    t0 = min(r[3] for r in g)
    st = [(r[3] - t0) / 1e3 for r in g]
    en = [(r[4] - t0) / 1e3 for r in g]
    du = [(r[4] - r[3]) / 1e3 for r in g]
    sms = sorted(set(r[2] for r in g))
    slow = sorted(g, key=lambda r: r[4] - r[3])[-4:]
    print(f"launch: {len(g)} CTAs on {len(sms)} SMs | start p50 {q(st, .5):.1f} p90 {q(st, .9):.1f} max {max(st):.1f}"
          f" | end p10 {q(en, .1):.1f} p50 {q(en, .5):.1f} p90 {q(en, .9):.1f} max {max(en):.1f}"
          f" | dur p10 {q(du, .1):.1f} p50 {q(du, .5):.1f} max {max(du):.1f} us | slowest (blk,z,sm): "
          + " ".join(f"({r[0]},{r[1]},{r[2]})" for r in slow))
