"""CPU ORACLE for GROUTER's data-passing hot path -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct Python + NumPy restatement of what the method
computes, following PAPER.md (marker text of Wu et al.,
EuroSys '26).  Each function cites the passage it follows as ``L<line> §<sec>``.

* Devices are simulated: every device buffer is a NumPy ``uint8`` array and
  every copy is ``np.copyto`` (memcpy).  Delivered bytes are pinned by
  identity: get(put(x)) == x.
* Decisions (placement, chunk split, tenant order, victims) follow the paper's
  algorithm step by step with integer arithmetic only (R30).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares NO code with
``paper_conf_eurosys_wulywdyfwwj26_b200`` (the CUDA path) and never imports it.

Parity status per function:
  splitter.plan_h2d / plan_single   pinned (brute force, worked example L242, tiling)
  routes.route_set / uplink_groups  pinned (worked example L178 Fig. 5a, special cases)
  stride.StrideServer               pinned (textbook stride bound I5, work conservation,
                                    hand-computed golden log)
  model.Oracle                      pinned (identity, I1-I7 invariants, Fig. 11b worked
                                    example L258, hand-derived golden traces)
  model.auto_cap / refresh_cap (O10) pinned (closed forms by hand, hand-derived golden
                                    case G; the measured availability is an input)
"""
