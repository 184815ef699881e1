"""CPU oracle for the nested-pattern hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package.  It shares no code with ``paper_conf_micro_leebsro14_b200`` (the CUDA
path): no kernels, headers, helpers, tables or constants; both follow DESIGN.md.  Everything here is
plain and slow on purpose: fp64 / exact Python integers, NumPy used only as a library primitive
(a reduction), every function citing the PAPER.md passage it follows.

Modules
  sums    — sumRows / sumCols / Split(k) partials / weighted variants   (Fig 1 L68-70, L542-550, Fig 15)
  select  — nest descriptors, constraints, Algorithm 1, ControlDOP, R2  (§IV)
  kmeans  — k-means assignment (argmin of squared distances)            (BASELINE.json config 4)
  logreg  — batched logistic-regression gradient                        (BASELINE.json config 5)

Readings of points the paper leaves open: the soft-constraint intrinsic weights and the
tie-break key are pinned by invariance (every reading consistent with L674-676 / L741 gives the same
records on the BASELINE workloads); the R2 runtime rule by schedule properties (tests/test_r2_properties.py).
"""
