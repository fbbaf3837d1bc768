"""CPU oracle for the out-of-order backprop (ooo backprop) data-parallel hot path.

TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the C-ABI library
under ``paper_conf_eurosys_ohlks22_b200/`` and its Python binding) may import,
call, link or execute anything in this package.  The only legitimate callers
are ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs.

The oracle is a plain, slow, obviously-correct NumPy float64 transcription of
what the paper's method computes.  It shares no code with the CUDA path (no
common kernels, headers, helpers, tables or constants).

Citations ``P:N`` refer to line N of the paper text
(``/root/reference/PAPER.md``, Oh, Lee, Kim, Seo, "Out-Of-Order BackProp",
EuroSys'22), followed by the section / equation / algorithm it sits in.

Modules
-------
``layers``     forward / backward of a dense-layer stack, op-by-op execution of
               a backward schedule D, data-parallel averaging, bf16 storage
               rounding (§2, §3, §5.1).
``schedule``   Algorithm 2 (reverse first-k), the k memory clamp
               (the formula is garbled -- reading Q3) and the k
               heuristic search (prose only -- reading Q4).
``unit_sim``   unit-time list-scheduling simulator used to pin the dependency
               rules against the paper's worked examples (Fig. 4, P:164/P:180/
               P:206; Fig. 5, P:226/P:232/P:236).

Pin status: every function is pinned by a
``-m "not gpu"`` test against something other than itself.
``schedule.max_k`` and ``schedule.search_k`` are pinned to their readings
(Q3, Q4: the paper gives no numeric example, so the readings themselves rest
on the text alone) by traces expanded by hand from the readings' wording
(tests/golden/alg2_kclamp_ksearch.json).
"""
