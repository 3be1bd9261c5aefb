"""Summarise gpurun_out/parity/*.json (written by the GPU parity tests through
tests/parity_metrics.py) into a markdown table: per case the loss error, the
worst per-tensor inf-norm and 2-norm errors, and every tensor above 2e-2 with
its bf16-storage-emulation error (the bound it is held to)."""
import glob
import json
import os
import sys

src = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/parity"
rows = []
for f in sorted(glob.glob(os.path.join(src, "*.json"))):
    d = json.load(open(f))
    g = [r for r in d["grads"] if not r.get("zero")]
    z = [r for r in d["grads"] if r.get("zero")]
    worst = max(g, key=lambda r: r["inf"])
    w2 = max(g, key=lambda r: r["rel2"])
    over = [r for r in g if r["inf"] > (1e-4 if d["dtype"] == "fp32" else 2e-2)]
    rows.append((d["case"], d["dtype"], d.get("hidden"), d.get("n_layers"), d["loss_rel"], worst, w2, over, z))
print("| case | dtype | H | L | loss rel err | worst inf-norm (tensor) | worst rel 2-norm (tensor) | "
      "tensors > bound: inf / bf16-storage emulation | provably-zero tensors |")
print("|---|---|---|---|---|---|---|---|---|")
for case, dt, H, L, lr, w, w2, over, z in rows:
    ov = "; ".join(f"{r['name']} {r['inf']:.4f} / {r.get('emulated_inf', float('nan')):.4f}" for r in over) or "-"
    zz = ", ".join(r["name"] for r in z) or "-"
    print(f"| {case} | {dt} | {H} | {L} | {lr:.1e} | {w['inf']:.4f} ({w['name']}) | {w2['rel2']:.4f} ({w2['name']}) "
          f"| {ov} | {zz} |")
