"""BAT oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct fp64 CPU implementation of what the Bipartite Attention
prefill computes, written from the paper text (/root/reference/PAPER.md, cited as P:<line>)
and the readings listed in DESIGN.md §"Readings of the paper".  It shares no code with the
CUDA path (paper_conf_asplos_0017wzlxszh0w26_b200/): no kernels, headers, helpers,
tables or constant generators; the two only share the seeded input generators in
``synth/``, which hold none of the method's arithmetic.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / reference
leg may import anything under ``oracle/``.  The product path never does.

Modules
-------
sequence   prompt ordering, segment ids, bipartite positions and the explicit T x T mask
           (§4.2; Fig. 1 caption P:131)
model      Qwen2-shaped transformer forward in fp64: full recompute (the plain definition,
           P:169-171) and the prefix-cached variant (§3.2); entity KV precompute
           
score      discriminant logits, softmax over the N item identifiers, TopK (§2.2)
plan       the integer plan (positions, segments, page tables, key metadata, tile states)
           by brute force
attention  single-layer masked attention over explicit key sets
hrcs       Algorithm 1 HRCS placement
scheduler  hotness-aware prefix selection rule
sizes      KV-cache size model (Table 2)

Pins: every function is pinned by ``tests/test_oracle_*.py`` (``-m "not gpu"``) against
closed forms, brute force, a library routine (HuggingFace transformers Qwen2) or values the
paper prints.  The UP-vs-IP score difference in the general case has no pin ("parity
unpinned") — the paper gives no formula relating them (SURVEY §8(c) issue 1).
"""
