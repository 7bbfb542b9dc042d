"""Summarise an ncu launch list (--csv --log-file) of one bench step.

usage: launch_summary.py launches.csv N_PER_STEP [--json traffic.json]
Groups the first N_PER_STEP launches (one step) by kernel, prints a markdown
table (time share, DRAM bytes if the capture has dram__bytes_*), and with
--json writes {kernel_class: dram_bytes_per_step} for bench.py's roofline.
ncu times are cold-cache and serialised: compare SHARES with bench.py's live
per-class times, not absolute values.
"""
import collections, csv, io, json, sys

CLASS = {"tc_chain_kernel": "tc_chain", "tc_wide_kernel": "tc_chain_wide", "conv_tc_kernel": "tc_conv", "conv_tma_kernel": "tc_conv",
         "conv_small_kernel": "simt_conv_small", "conv_stem_kernel": "mma_conv_stem", "linear_kernel": "simt_linear", "conv_kernel": "simt_conv",
         "ew_kernel": "simt_ew", "group_simt_kernel": "simt_group", "group_gap_kernel": "simt_group_gap",
         "mma_chain_kernel": "mma_chain", "mma_lean_kernel": "mma_lean", "conv_rank_mma_kernel": "mma_conv_rank", "mma_catp_kernel": "mma_catp",
         "conv_rank_kernel": "simt_conv_rank", "dwconv_vec_kernel": "simt_dwconv_vec", "gemm_kernel": "tc_gemm", "tile_conv_kernel": "mma_conv_tile", "dwpair_kernel": "simt_dwpair", "dwpair_generic_kernel": "simt_dwpair", "gemm_reduce_kernel": "tc_gemm", "pair_chain_kernel": "tc_pair",
         "mma_lean64_kernel": "mma_lean", "mma_poolcat_kernel": "mma_poolcat", "mma_cat_kernel": "mma_cat",
         "dwconv_col_kernel": "simt_dwconv_vec", "dwconv_row_kernel": "simt_dwconv_vec"}

path, n = sys.argv[1], int(sys.argv[2])
lines = open(path).read().splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
launch = collections.OrderedDict()
for r in rows:
    d = launch.setdefault(int(r["ID"]), {"name": r["Kernel Name"]})
    v = r["Metric Value"].replace(",", "")
    try:
        d[r["Metric Name"]] = float(v)
    except ValueError:
        pass
def short(name):
    n = name.split("(")[0].split("::")[-1]
    return n.split("<")[0].split(" ")[-1]


ids = [i for i in sorted(launch) if short(launch[i]["name"]) in CLASS][:n]   # our kernels only
agg = collections.OrderedDict()
for i in ids:
    d = launch[i]
    k = short(d["name"])
    a = agg.setdefault(k, {"n": 0, "ns": 0.0, "dram": 0.0})
    a["n"] += 1
    a["ns"] += d.get("gpu__time_duration.sum", 0.0)
    a["dram"] += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
tot = sum(a["ns"] for a in agg.values())
print(f"| kernel | launches | total us | share | DRAM MB |")
print("|---|---:|---:|---:|---:|")
for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["ns"]):
    print(f"| {k} | {a['n']} | {a['ns'] / 1e3:.1f} | {100 * a['ns'] / tot:.1f}% | {a['dram'] / 1e6:.1f} |")
print(f"| total | {len(ids)} | {tot / 1e3:.1f} | 100% | {sum(a['dram'] for a in agg.values()) / 1e6:.1f} |")
if "--json" in sys.argv:
    out = collections.defaultdict(float)
    for k, a in agg.items():
        out[CLASS.get(k, k)] += a["dram"]
    json.dump(dict(out), open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)
