"""profiles/ncu_traffic.json from a round's ncu_full_summary.json: per (kernel,
variant) capture, dram__bytes_read.sum + dram__bytes_write.sum of that one
launch (bytes).  bench.py reports it as roofline.traffic for the dominant
kernel.  usage: traffic_from_summary.py SUMMARY.json OUT.json"""
import json
import sys

CAP = {"binarysearch": "binarysearch", "fwt_ps": "fwt", "prefixsum": "prefixsum", "reduction": "reduction",
       "transpose": "transpose", "sobel": "sobel", "dct": "dct", "matmul": "matmul", "blackscholes": "blackscholes",
       "fw_pass": "floydwarshall"}
VARIANTS = ("inter_group", "intra_smem", "intra_reg", "none")

summ = json.load(open(sys.argv[1]))
out = {}
for name, ms in summ.items():
    m = ms[0] if isinstance(ms, list) else ms  # one launch per capture
    for v in VARIANTS:
        if name.endswith("_" + v):
            cap = name[: -len(v) - 1]
            if cap in CAP and "dram_read_MB" in m and "dram_write_MB" in m:
                out[f"{CAP[cap]}/{v}"] = int(round((m["dram_read_MB"] + m["dram_write_MB"]) * 1e6))
            break
json.dump(dict(sorted(out.items())), open(sys.argv[2], "w"), indent=0)
print(len(out), "entries")
