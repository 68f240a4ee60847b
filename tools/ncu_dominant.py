"""Write profiles/ncu_dominant.json (the per-algorithmic-byte DRAM traffic of the dominant kernel
that bench.py scales into its roofline `traffic`) from an ncu summary json of a C3 capture.

    python tools/ncu_dominant.py profiles/rXX_ncu.json"""
import json, sys

src = sys.argv[1]
d = json.load(open(src))
k = [k for k in d["kernels"] if "p3_kernel<float, 8, 8, 8" in k["kernel"]][0]
alg = 2 * 512 ** 3 * 4
rd, wr = k["dram_read_bytes"], k["dram_write_bytes"]
out = {"kernel_pattern": "P3_ssim", "kernel": k["kernel"],
       "workload": "C3-nyx-512^3 (ncu --set full, kernel replay; the C5 pair is too large to save/restore for replays)",
       "source": [src], "dram_bytes_per_launch_C3": rd + wr, "dram_read_bytes_C3": rd, "dram_write_bytes_C3": wr,
       "algorithmic_bytes_C3": alg, "dram_bytes_per_alg_byte": (rd + wr) / alg, "duration_us_cold_C3": k["duration_us"]}
json.dump(out, open("profiles/ncu_dominant.json", "w"), indent=1)
print(json.dumps(out, indent=1))
