"""SLO-derived tenant shares (reading R43).

TEST INFRASTRUCTURE ONLY: imported by tests/, smoke() and bench.py's
cpu_baseline leg; never by the product path.

Paper basis (§4.3.2 "Transfer rate control", L193-L197, L227):
* "Rate_least is defined as data_size / (L_slo - L_infer)" -- the minimum
  transfer rate that still meets the function's SLO.
* "Rate_idle = BW_all - sum_i Rate_least^i" -- the bandwidth left once every
  function's minimum is met.
* "GROUTER allocates this idle bandwidth to the function with the tightest
  SLO" (L227).
* chunks are scheduled "proportionally" to the allocated bandwidth (L193),
  i.e. the allocation becomes the stride weight of the tenant (O8, R7).

Reading R43 (integer arithmetic, stated in DESIGN.md):
  Rate_least = ceil(data_bytes * 10^9 / (slo_ns - infer_ns))   [B/s]
  BW_all     = sum of the calibrated solo host->GPU rates h2d_Bps
  Rate_idle  = max(0, BW_all - sum Rate_least)
  rate_t     = Rate_least_t + (Rate_idle if t has the tightest SLO: min slo_ns,
               ties -> lower workflow id)
  weight_t   = min(2^32 - 1, max(1, ceil(rate_t / 2^20)))     [MiB/s units]
"""
from __future__ import annotations

NS = 10 ** 9
UNIT = 1 << 20
WMAX = (1 << 32) - 1


def rate_least(data_bytes: int, slo_ns: int, infer_ns: int) -> int:
    """Rate_least = data_size / (L_slo - L_infer) (L195), rounded up, B/s."""
    if slo_ns <= infer_ns:
        raise ValueError("SLO not above the inference latency: no transfer rate meets it")
    return -(-(data_bytes * NS) // (slo_ns - infer_ns))


def rate_idle(bw_all: int, least: list) -> int:
    """Rate_idle = BW_all - sum Rate_least (L197), floored at 0."""
    return max(0, bw_all - sum(least))


def tightest(slos: dict) -> int:
    """Tenant with the tightest SLO (L227): min slo_ns, ties -> lower id."""
    return min(slos, key=lambda wf: (slos[wf][1], wf))


def allocate(slos: dict, bw_all: int) -> dict:
    """slos: wf -> (data_bytes, slo_ns, infer_ns).  Returns wf -> rate (B/s)."""
    if not slos:
        return {}
    least = {wf: rate_least(*v) for wf, v in slos.items()}
    idle = rate_idle(bw_all, list(least.values()))
    t = tightest(slos)
    return {wf: least[wf] + (idle if wf == t else 0) for wf in slos}


def weights(slos: dict, bw_all: int) -> dict:
    """Stride weights from the allocated rates, in MiB/s (R43)."""
    return {wf: min(WMAX, max(1, -(-r // UNIT))) for wf, r in allocate(slos, bw_all).items()}
