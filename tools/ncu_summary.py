"""Summarise an ncu report (raw page) or a launch-list CSV into markdown for profiles/."""
import csv, collections, re, subprocess, sys

KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "launch__grid_size",
        "launch__block_size", "launch__registers_per_thread", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "sm__ops_path_tensor_op_utcimma_src_int8_sparsity_off.sum",
        "sm__ops_path_tensor_op_utcimma_src_int8_sparsity_off.sum.per_second",
        "sm__ops_path_tensor_op_utcimma_src_int8_sparsity_off.sum.peak_sustained_elapsed.per_second",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]


def rep(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    lines = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        lines.append(f"### `{d.get('Kernel Name', '')[:120]}`\n")
        lines.append("| metric | value | unit |\n|---|---|---|")
        for k in KEYS:
            if k in d and d[k] not in ("", "n/a"):
                lines.append(f"| {k} | {d[k]} | {units[hdr.index(k)]} |")
        stalls = [(k, d[k]) for k in hdr if "pcsamp_warps_issue_stalled" in k and not k.endswith("not_issued")
                  and d[k] not in ("", "n/a", "0")]
        stalls.sort(key=lambda x: -float(x[1].replace(",", "")))
        if stalls:
            lines.append("\nTop warp stall samples: " + ", ".join(f"{k.split('stalled_')[1]}={v}" for k, v in stalls[:6]))
        lines.append("")
    return "\n".join(lines)


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            name = re.sub(r"\(.*", "", d["Kernel Name"])[:100]
            agg[name][0] += 1
            agg[name][1] += float(d["Metric Value"])
    tot = sum(v[1] for v in agg.values())
    lines = ["| kernel | launches | total us | share | avg us |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k}` | {v[0]} | {v[1] / 1e3:.1f} | {100 * v[1] / tot:.1f}% | {v[1] / v[0] / 1e3:.2f} |")
    return "\n".join(lines)


if __name__ == "__main__":
    p = sys.argv[1]
    print(launches(p) if p.endswith(".csv") else rep(p))
