"""Markdown table of the committed G = 1 bench lines (profiles/r02_bench_<config>_g1.json), so the
tables in DESIGN.md / README.md / profiles/README.md are regenerated, not retyped.

  python scripts/bench_table.py [design|readme]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ROUND = "r02"
ROWS = [("swin_b", "Swin-B, N=32 (headline)"), ("resnet50", "ResNet-50, N=8"), ("vgg19", "VGG-19, N=16"), ("bert_base", "BERT bf16, N=12"),
        ("tiny", "tiny, N=4")]


def main(kind="design"):
    out = []
    if kind == "design":
        out.append("| config | step ms | EST-gradient GB/s | k_fold frac | k_stash frac (phase) | step frac "
                   "(of nominal 8 TB/s) | e2e GB/s (frac of H2D) | NEXT-1 tail ms (copy tail) | parity |")
        out.append("|---|---|---|---|---|---|---|---|---|")
    else:
        out.append("| config | step (stash + switch + fold) | EST-gradient GB/s | k_fold vs measured HBM peak |")
        out.append("|---|---|---|---|")
    for name, label in ROWS:
        with open(os.path.join(ROOT, "profiles", f"{ROUND}_bench_{name}_g1.json")) as f:
            d = json.load(f)
        r = d["roofline_by_kernel"]
        p = d["parity"]
        par = "whole output = oracle (SHA-256)" if p.get("full_output_checked") and p.get("sha256_equal") \
            else "sampled windows bit-exact"
        if kind == "design":
            out.append(f"| {label} | {d['ms_per_step']:.3f} | {d['value']:.0f} | {r['k_fold']['frac']:.2f} | "
                       f"{r['k_stash']['frac']:.2f} | {d['step_roofline']['frac']:.2f} "
                       f"({d['step_roofline']['frac_of_nominal']:.2f}) | {d['e2e']['value']:.1f} "
                       f"({d['e2e']['roofline']['frac']:.2f}) | {d['next1']['tail_ms']:.3f} "
                       f"({d['next1']['copy_step_tail_ms']:.3f}) | {par} |")
        else:
            out.append(f"| {label} | {d['ms_per_step']:.3f} ms | {d['value']:.0f} | {r['k_fold']['frac']:.2f} |")
    print("\n".join(out))


if __name__ == "__main__":
    main(*sys.argv[1:])
