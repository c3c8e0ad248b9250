"""Traces of the hand-derived eviction-branch cases (tests/golden/eviction_branches.md).

Inputs only: each builder returns (ops, run kwargs).  Every case ends with a
flush (replay mode dispatches queued copies only there; it moves no
placement, victim or accounting).  The expected values live
in tests/golden/eviction_branches.json, typed in by hand from the derivation;
the oracle is checked against them (tests/test_oracle_branches.py) and the
library against the oracle on the GPU (tests/test_gpu_parity.py).
"""
from synth import traces as T

MiB = 1 << 20


def case_a():
    """R15: mixed hinted / unhinted victims."""
    b = T.Builder(21)
    f, g = T.fn(1, 1, 0), T.fn(1, 2, 0)
    A, B, C, D, E = (b.put(f, MiB) for _ in range(5))      # ops 0-4
    b.next_use(A, 3)                                        # 5
    b.next_use(C, 7)                                        # 6
    b.next_use(E, 7)                                        # 7
    b.get_into(g, B)                                        # 8
    b.put(f, 5 * MiB)                                       # 9
    b.put(f, MiB)                                           # 10
    o8 = b.put(f, 3 * MiB)                                  # 11
    o9 = b.put(f, 1)                                        # 12
    b.next_use(o8, 5)                                       # 13
    b.next_use(o9, 0)                                       # 14
    b.put(f, 3 * MiB)                                       # 15
    b.flush()                                               # 16 (replay: dispatch)
    del D
    return b.ops, {"pool_cap": [10 * MiB], "host_store_bytes": 1 << 30}


def case_b():
    """R33 all-or-nothing reserve, R16 put -> host store, alloc -> ENOMEM."""
    b = T.Builder(22)
    f, z, c = T.fn(1, 1, 0), T.fn(1, 2, 0), T.fn(1, 3, T.HOST)
    o1 = b.put(f, 3 * MiB)                                  # 0
    b.get(z, o1)                                            # 1 zero copy pin
    b.put(f, MiB)                                           # 2
    b.put(c, 5 * MiB, hint=0)                               # 3
    b.alloc(f, 5 * MiB)                                     # 4
    b.put(f, MiB)                                           # 5
    b.flush()                                               # 6 (replay: dispatch)
    return b.ops, {"pool_cap": [6 * MiB], "host_store_bytes": 64 * MiB}


def case_c():
    """R34: set_pool_limit below the unevictable floor."""
    b = T.Builder(23)
    f, z = T.fn(1, 1, 0), T.fn(1, 2, 0)
    o1 = b.put(f, 3 * MiB)                                  # 0
    g = b.get(z, o1)                                        # 1
    b.put(f, 3 * MiB)                                       # 2
    b.put(f, MiB)                                           # 3
    b.pool_limit(0, 2 * MiB)                                # 4
    b.put(f, 1)                                             # 5
    b.release(z, g)                                         # 6
    b.pool_limit(0, 2 * MiB)                                # 7
    b.flush()                                               # 8 (replay: dispatch)
    return b.ops, {"host_store_bytes": 64 * MiB}


def case_d():
    """R32: host store full."""
    b = T.Builder(24)
    c, g, r = T.fn(1, 1, T.HOST), T.fn(1, 2, 0), T.fn(1, 3, T.HOST)
    o1 = b.put(c, 3 * MiB)                                  # 0
    b.put(c, 1)                                             # 1
    b.alloc(c, 1)                                           # 2
    o2 = b.put(g, MiB)                                      # 3
    b.get(r, o2)                                            # 4
    b.put(g, MiB)                                           # 5
    b.get_into(r, o2)                                       # 6
    b.free(c, o1)                                           # 7
    b.put(c, 1)                                             # 8
    b.put(g, MiB)                                           # 9
    b.flush()                                               # 10 (replay: dispatch)
    return b.ops, {"pool_cap": [2 * MiB], "host_store_bytes": 4 * MiB}


def case_e():
    """Status rules of the boundary (SURVEY §8(b) conventions, R19, R35)."""
    b = T.Builder(25)
    g, other = T.fn(1, 1, 0), T.fn(2, 1, 0)
    o1 = b.alloc(g, MiB)                                    # 0 OPEN
    b.free(g, o1)                                           # 1 EBUSY
    b.get(g, o1)                                            # 2 ENOENT (unsealed)
    b.seal(other, o1)                                       # 3 EPERM
    b.seal(g, o1)                                           # 4
    b.seal(g, o1)                                           # 5 ESTATE
    b.get_into(g, o1, cap=MiB - 1)                          # 6 EINVAL
    z = b.get(g, o1)                                        # 7 zero copy
    b.release(other, z)                                     # 8 EPERM
    b.free(other, o1)                                       # 9 EPERM
    b.weight(1, 0)                                          # 10 EINVAL
    b.next_use(1, 5)                                        # 11 ENOENT (op 1 created nothing)
    b.pool_limit(3, 0)                                      # 12 EINVAL (one GPU)
    b.release(g, z)                                         # 13
    b.free(g, o1)                                           # 14
    b.get(g, o1)                                            # 15 ENOENT (freed)
    b.flush()                                               # 16
    return b.ops, {"host_store_bytes": 64 * MiB}


def case_f():
    """Placement rules (R23, R38; PAPER.md L165 locality): two GPUs."""
    b = T.Builder(26)
    g0, c, g1 = T.fn(1, 1, 0), T.fn(1, 2, T.HOST), T.fn(1, 3, 1)
    o1 = b.put(g0, MiB, hint=1)                             # 0 gFn put: local, hint ignored
    b.put(c, MiB, hint=1)                                   # 1 cFn put with a hint: staged to GPU1
    b.put(c, MiB)                                           # 2 cFn put without a hint: host store
    b.alloc(c, MiB, hint=1)                                 # 3 cFn alloc: caller's location (host)
    b.alloc(g0, MiB, hint=1)                                # 4 gFn alloc: its own GPU
    b.get(g1, o1)                                           # 5 another GPU: copy lease on GPU1
    b.flush()                                               # 6
    return b.ops, {"host_store_bytes": 64 * MiB, "n_gpus": 2}


def case_g():
    """O10 auto cap (L262 "triggers data migration and restoration
    automatically based on available GPU memory ... 50% of free memory";
    R12, R54) with proactive restore (R42)."""
    b = T.Builder(27)
    f, g = T.fn(1, 1, 0), T.fn(1, 2, 0)
    A = b.put(f, 3 * MiB)                                   # 0
    B = b.put(f, MiB)                                       # 1
    b.put(f, MiB)                                           # 2 C, no hint
    b.next_use(A, 2)                                        # 3
    b.next_use(B, 5)                                        # 4
    b.refresh_cap(0, 9 * MiB + 123)                         # 5 cap 4 MiB
    b.refresh_cap(0, 12 * MiB)                              # 6 cap 6 MiB
    b.refresh_cap(0, 3 * MiB)                               # 7 cap 0
    b.refresh_cap(5, MiB)                                   # 8 EINVAL (one GPU)
    b.get_into(g, B)                                        # 9 from the host store
    b.refresh_cap(0, 100 * MiB + 1)                         # 10 cap 50 MiB
    b.flush()                                               # 11
    return b.ops, {"host_store_bytes": 64 * MiB, "restore": True}


CASES = {"A": case_a, "B": case_b, "C": case_c, "D": case_d, "E": case_e, "F": case_f, "G": case_g}
