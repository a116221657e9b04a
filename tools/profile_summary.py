"""Write profiles/TAG_summary.md (+ TAG_traffic.json, TAG_ring_traffic.json) from a tools/gpu/bench.sh
run's outputs in gpurun_out/ (TAG_bench.json, TAG_launches.csv, TAG_full.ncu-rep, TAG_ring4096.ncu-rep),
and copy the bench line and launch list into profiles/.

    python tools/profile_summary.py r02f "one-line description of the code state"
"""
import json
import os
import shutil
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import ncu_summary  # noqa: E402

tag = sys.argv[1]
what = sys.argv[2] if len(sys.argv) > 2 else ""
G, P = "gpurun_out", "profiles"
line = open(f"{G}/{tag}_bench.json").read().strip().splitlines()[-1]
d = json.loads(line)
shutil.copy(f"{G}/{tag}_bench.json", f"{P}/{tag}_bench.json")
shutil.copy(f"{G}/{tag}_launches.csv", f"{P}/{tag}_launches.csv")
here = os.path.dirname(os.path.abspath(__file__))
subprocess.run([sys.executable, f"{here}/traffic.py", f"{G}/{tag}_full.ncu-rep", f"{P}/{tag}_traffic.json"],
               capture_output=True)
subprocess.run([sys.executable, f"{here}/traffic.py", f"{G}/{tag}_ring4096.ncu-rep", f"{P}/{tag}_ring_traffic.json"],
               capture_output=True)
rg = {(r["n"], r["l"]): r for r in d.get("ring_gemm", [])}
c1 = d.get("beaver_matmul_cfg1", {})
out = [f"# Profiles {tag}: {what}\n",
       f"Bench line `{tag}_bench.json` (default `python bench.py`, 1 x B200, clocks "
       f"{d['clocks'].get('sm_mhz')} MHz median over the whole bench, reasons {d['clocks'].get('reasons')}): "
       f"**{d['value']:,.0f} samples/s** secure MLP training (ms/step {d['ms_per_step']:.4f}), "
       f"e2e {d['e2e']['value']:,.0f}, online graph {d.get('online_graph_samples_per_s') or 0:,.0f}, "
       f"online (eager) {d.get('online_samples_per_s') or 0:,.0f}, inference {d.get('infer_samples_per_s') or 0:,.0f}."]
if rg:
    a, b = rg.get((4096, 64)), rg.get((4096, 32))
    out.append(f"Ring GEMM 4096^3 l=64 {a['ms']:.3f} ms = {a['useful_limb_tops']:.0f} useful TOPS = "
               f"{a['roofline']['frac']:.3f} of the INT8 ceiling measured in the same run ({a['roofline']['peak']:.0f} TOPS); "
               f"l=32 {b['ms']:.3f} ms ({b['roofline']['frac']:.3f}).")
if c1:
    out.append(f"Config 1 (one Beaver matmul 128x784 . 784x1): {c1['p50_us']:.1f} us p50 in {c1['launches_per_call']} "
               f"launch(es), bit-exact {c1['bitexact_vs_oracle']} (oracle {c1['oracle_us_per_call']:.0f} us).")
out.append(f"\nFiles: `{tag}_launches.csv` (`ncu --metrics gpu__time_duration.sum --clock-control none` launch list of "
           f"`bench.py --steps 20 --warmup 3 --no-ring-gemm --no-cpu-baseline --no-classes --no-secondary`: cold "
           f"cache, serialised -- shares, not absolute times); `{tag}_traffic.json` (per-class DRAM bytes per launch from "
           f"the `--set full` capture of the step kernels; the report itself stays out of the tree, its metrics are "
           f"below); `{tag}_ring_traffic.json` (`--set full` of one 4096^3 l=64 ring GEMM).\n")
kc = d.get("kernel_classes") or {}
if kc:
    out.append("## Kernel classes of the MLP step (CUPTI, attributed along the PDL chain)\n")
    out.append("| class | us / step | launches / step | us / launch | share of online step |\n|---|---|---|---|---|")
    for k, v in kc.items():
        if k.startswith("_"):
            continue
        out.append(f"| {k} | {v['ms_per_step'] * 1e3:.1f} | {v['launches_per_step']:g} | "
                   f"{v['ms_per_launch'] * 1e3:.2f} | {100 * v.get('share_of_online_step', 0):.0f}% |")
rf = d.get("roofline") or {}
if rf:
    out.append(f"\nRoofline of the dominant class (`{rf.get('class')}`, {rf.get('kernel')}): {rf['achieved']:.0f} "
               f"{rf['unit']} per launch = **{rf['frac']:.3f}** of {rf['peak']:.0f} ({rf.get('peak_source')}).")
si = d.get("step_int8_fraction") or {}
if si:
    out.append(f"Whole step: {si['achieved_tops']:.1f} useful TOPS = {si['frac']:.4f} of the INT8 ceiling.")
off = d.get("offline") or {}
if off:
    out.append(f"Offline (the dealer alone): {off['ms_per_step'] * 1e3:.1f} us/step, "
               f"{off['prg_alu_roofline']['frac_lower_bound']:.3f} of the ChaCha20 ALU roofline.")
out.append("\n## Launch list (ncu, serialised, cold cache)\n")
out.append(ncu_summary.launches(f"{G}/{tag}_launches.csv"))
out.append("\n## ncu --set full: step kernels\n")
out.append(ncu_summary.rep(f"{G}/{tag}_full.ncu-rep"))
out.append("\n## ncu --set full: 4096^3 ring GEMM\n")
out.append(ncu_summary.rep(f"{G}/{tag}_ring4096.ncu-rep"))
open(f"{P}/{tag}_summary.md", "w").write("\n".join(out) + "\n")
print(f"wrote {P}/{tag}_summary.md")
