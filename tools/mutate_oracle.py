"""Mutation check of the oracle pins (VERDICT r01 Next #1 "Done" criterion).

Applies one-line mutations to oracle/model.py, one at a time, runs the pin
tests that should catch each, and restores the file.  Every mutation must
turn at least one pin red.  Usage: python tools/mutate_oracle.py
"""
from __future__ import annotations

import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MODEL = os.path.join(ROOT, "oracle", "model.py")
PINS = ["tests/test_oracle_branches.py", "tests/test_oracle_model.py"]

# (what it breaks, original line, mutated line)
MUTATIONS = [
    ("R15 hinted objects first", "        return sorted(cs, key=lambda o: (0 if o.next_use is None else 1,",
     "        return sorted(cs, key=lambda o: (1 if o.next_use is None else 0,"),
    ("R15 ascending next-use", "                                         0 if o.next_use is None else -o.next_use,",
     "                                         0 if o.next_use is None else o.next_use,"),
    ("R15 MRU instead of LRU", "                                         o.last_access, o.oid))",
     "                                         -o.last_access, o.oid))"),
    ("R33 no feasibility check (partial eviction)", "        if freed < need or self.host_used + freed > self.H:",
     "        if False:"),
    ("R33/R32 eviction ignores host room", "        if freed < need or self.host_used + freed > self.H:",
     "        if freed < need:"),
    ("R16 put fails instead of going to the host", "            home = HOST                                   # R16 spill on arrival",
     "            return ENOMEM, {}"),
    ("R34 limit reports OK when unmet", "        return (OK if self.used[d] <= self.cap[d] else ENOMEM), {}",
     "        return OK, {}"),
    ("R34 cap not kept when unreachable", "        self.cap[d] = nbytes",
     "        self.cap[d] = nbytes if sum(charge(o.n) for o in self._candidates(d)) >= self.used[d] - nbytes else self.cap[d]"),
    ("R32 host admission >=", "        if self.host_used + c > self.H:", "        if self.host_used + c >= self.H:"),
    ("R32 host leases not charged", "            ok = self._host_reserve(c) if d == HOST else self._reserve(d, c)",
     "            ok = True if d == HOST else self._reserve(d, c)"),
    ("seal twice accepted", "            return ESTATE, {}", "            pass"),
    ("free of an OPEN object -> ENOENT", "            return EBUSY, {}", "            return ENOENT, {}"),
    ("get_into accepts dst_cap = n - 1", "        if cap < o.n or (dst is None and o.n > 0):",
     "        if cap < o.n - 1 or (dst is None and o.n > 0):"),
    ("weight 0 accepted", "        if w < 1:", "        if w < 0:"),
    ("R35 release of a pin skips the workflow check", '            if o.wf != fn["wf"]:', "            if False:"),
    ("R23 gFn put follows its hint", "            home = dev", "            home = hint if hint >= 0 else dev"),
    ("R23 cFn hint ignored", "        elif hint >= 0:", "        elif False:"),
    ("O10 threshold rounded up", "    return avail * permille // 1000 // PAGE * PAGE",
     "    return -(-(avail * permille // 1000) // PAGE) * PAGE"),
    ("O10 whole availability, not half", "    return avail * permille // 1000 // PAGE * PAGE",
     "    return avail // PAGE * PAGE"),
    ("O10 no rounding to pages", "    return avail * permille // 1000 // PAGE * PAGE",
     "    return avail * permille // 1000"),
    ("R38 alloc follows the hint", "        home = dev\n        if home != HOST:",
     "        home = hint if hint >= 0 else dev\n        if home != HOST:"),
]


def main() -> int:
    orig = open(MODEL).read()
    rows, bad = [], 0
    try:
        for what, a, b in MUTATIONS:
            assert orig.count(a + "\n") == 1, f"mutation anchor not unique: {a!r}"
            open(MODEL, "w").write(orig.replace(a + "\n", b + "\n"))
            r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider"] + PINS,
                               cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
            failed = [ln.split(" ")[1] for ln in r.stdout.splitlines() if ln.startswith("FAILED")]
            caught = r.returncode != 0
            bad += not caught
            rows.append((what, "caught" if caught else "SURVIVED", failed[0] if failed else ""))
    finally:
        open(MODEL, "w").write(orig)
    for what, res, t in rows:
        print(f"{res:9s} {what:48s} {t}")
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
