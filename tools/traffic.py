"""Per-kernel-class DRAM traffic per launch from an ncu --set full report (for bench.py's roofline).

    python tools/traffic.py profiles/r01d_full.ncu-rep profiles/r01d_traffic.json

Maps kernel names to bench.py's kernel classes and averages dram__bytes_read.sum +
dram__bytes_write.sum over the captured launches of each class.
"""
import csv
import json
import subprocess
import sys

CLASSES = [("seg_gemm_kernel", "ring_gemm_cuda_core"), ("tc_seg_kernel", "ring_gemm_tcgen05"),
           ("msb_chain_pair_kernel", "msb_relu_eq9_rounds"), ("had_fused_kernel", "hadamard_rounds"),
           ("deal_prg_kernel", "dealer"), ("ring_gemm_cl_grouped", "dealer"), ("open_list_kernel", "beaver_mask"),
           ("tc_ring_gemm64_v4", "ring_gemm_tc_l64"), ("tc_ring_gemm_kernel", "ring_gemm_tc_l32"),
           ("split_kernel", "ring_gemm_limb_split")]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}

rep, out = sys.argv[1], sys.argv[2]
rows = list(csv.reader(subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                                      text=True).stdout.splitlines()))
hdr, units = rows[0], rows[1]
acc = {}
for r in rows[2:]:
    d = dict(zip(hdr, r))
    cls = next((c for k, c in CLASSES if k in d.get("Kernel Name", "")), None)
    if cls is None:
        continue
    b = 0.0
    for key in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        b += float(d[key].replace(",", "")) * SCALE.get(units[hdr.index(key)], 1)
    acc.setdefault(cls, []).append(b)
res = {c: {"bytes_per_launch_avg": sum(v) / len(v), "launches_captured": len(v)} for c, v in acc.items()}
res["source"] = f"{rep} (ncu --set full, cold cache): dram__bytes_read.sum + dram__bytes_write.sum"
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(res, indent=1))
