"""Render tools/sensitivity.py's JSON as the tables of profiles/<round>/f1_f4_sensitivity.md.
usage: python tools/sensitivity_md.py sensitivity.json > f1_f4_sensitivity.md"""
import json
import sys

d = json.load(open(sys.argv[1]))
print("# Row f1 (Fig. 11-12 analog) and f4 (Fig. 7 analog) on one B200\n")
print("Source: `tools/sensitivity.py`, SSSP from vertex 0 on seeded R-MAT graphs. A graph named \"i_j\" has about "
      "i M edges and j M vertices (PAPER.md L489). Times are the median `run_ms` of 3 runs to convergence, with the "
      "graph resident in HBM. Tables rendered by `tools/sensitivity_md.py`.\n")
print("## f1: G-Shards vs CW as windows shrink (paper: L473, L495, L497)\n")
print("| graph | \\|N\\| | shards | avg window (measured / model E·N²/V², L173) | GS ms (passes) | CW ms (passes) | GS / CW |")
print("|---|---|---|---|---|---|---|")
for r in d["f1"]:
    print(f"| {r['graph']} | {r['N']} | {r['S']} | {r['avg_window']} / {r['model_avg_window']} | "
          f"{r['gs_ms']:.3f} ({r['gs_passes']}) | {r['cw_ms']:.3f} ({r['cw_passes']}) | {r['gs_ms'] / r['cw_ms']:.2f} |")
print("\nThe full window-size histograms (0..128 entries, Fig. 11) are in the JSON (`window_hist_0_128`).\n")
print("## f4: per-pass committed updates (Fig. 7 analog, L433)\n")
for name, t in d["f4"].items():
    up, act = t["updated_vertices"], t["active_shards"]
    more = " ..." if len(up) > 8 else ""
    print(f"- **{name}** ({t['passes']} passes, {t['run_ms']:.2f} ms): updated vertices per pass {up[:8]}{more}; "
          f"active shards per pass {act[:8]}{more} of {t['num_shards']}")
