"""Summarise a per-work-item attention record (BAT_ATTN_ITEMS file: t_q t_s0 t_lastpv t_end kt_n cta
per work item, clock64 of the CTA's SM)."""
import sys
import numpy as np
it = np.loadtxt(sys.argv[1]).astype(np.int64)
it = it[it[:, 4] > 0]  # drop the planner's padding items
cta = it[:, 5]
print(f"work items {len(it)}  k-tiles mean {it[:,4].mean():.2f} min {it[:,4].min()} max {it[:,4].max()}")
span, per_tile, gaps, epi, head = [], [], [], [], []
for c in np.unique(cta):
    r = it[cta == c]
    r = r[np.argsort(r[:, 0])]
    span.append(r[-1, 3] - r[0, 0])
    per_tile += list((r[:, 2] - r[:, 1]) / np.maximum(1, r[:, 4] - 1))
    epi += list(r[:, 3] - r[:, 2])
    head += list(r[:, 1] - r[:, 0])
    gaps += list(r[1:, 0] - r[:-1, 2])
span = np.array(span)
tiles = np.array([it[cta == c][:, 4].sum() for c in np.unique(cta)])
print(f"CTA span (clk): mean {span.mean():.0f} min {span.min()} max {span.max()}  items/CTA {len(it)/len(span):.2f}"
      f"  k-tiles/CTA mean {tiles.mean():.1f} max {tiles.max()}  clk per k-tile (span/tiles) {np.mean(span / tiles):.0f}")
print(f"per item: q->S0 issued {np.mean(head):.0f}  S0..lastPV per k-tile {np.mean(per_tile):.0f}  "
      f"lastPV->epilogue done {np.mean(epi):.0f}  lastPV(i)->q_full(i+1) {np.mean(gaps):.0f}")
