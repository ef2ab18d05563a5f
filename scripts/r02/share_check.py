"""Bench roofline vs ncu launch list: each class's share of the step (bench: graph-profiled
per-class event timing; ncu: gpu__time_duration.sum of the eager step, cold-cache, serialised)
and the dominant kernel's frac recomputed from the ncu average launch time."""
import json, sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import summarize_launches as sl

bench, launches = sys.argv[1], sys.argv[2]
d = json.loads([l for l in open(bench) if l.startswith("{")][-1])
r = d["roofline"]
agg = sl.summarize(launches)
match = {"gemm_qkv": "linear_tc_kernel<2, 256, 0>", "gemm_ffn1": "linear_tc_kernel<2, 256, 2>",
         "gemm_ffn2": "linear_lng_kernel", "gemm_o": "linear_ln_kernel", "attention": "attn_tc3",
         "embed": "pack_embed_kernel", "unpack": "unpack_kernel"}
ours = {k: v for k, v in agg.items() if any(m in k for m in match.values())}
tot_n = sum(v[1] for v in ours.values())
tot_b = sum(v["ms_per_step"] for v in r["classes"].values())
print("%-10s %-34s %9s %9s %9s %9s" % ("class", "ncu kernel", "bench_sh", "ncu_sh", "bench_us", "ncu_us"))


def agg_class(c):
    """(launches, total us, names) over every ncu kernel of class c (e.g. both FFN2 variants:
    the last layer's fused-unpack instantiation and the others)."""
    ks = [k for k in ours if match[c] in k]
    return sum(ours[k][0] for k in ks), sum(ours[k][1] for k in ks), "+".join(ks)


for c, v in r["classes"].items():
    n, tot, name = agg_class(c)
    if n == 0:
        continue
    print("%-10s %-34s %9.4f %9.4f %9.2f %9.2f" % (c, name[:34], v["ms_per_step"] / tot_b, tot / tot_n,
                                                 v["us_per_launch"], tot / n))
n, tot, _ = agg_class(r["class"])
ncu_us = tot / n
print("dominant %s: bench frac %.4f (%.2f us per launch in the graph-timed step); frac from the ncu "
      "average launch (%.2f us, cold cache) %.4f" % (r["class"], r["frac"], r["us_per_launch"], ncu_us,
                                                      r["work_per_launch"] / (ncu_us * 1e-6) / 1e12 / r["peak"]))
