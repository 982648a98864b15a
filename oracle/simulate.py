"""O4 — tiled simulator of the customised matrix-based segmented sum
(TEST INFRASTRUCTURE ONLY, see oracle/__init__).  Pure Python loops, tiny inputs only.

Follows PAPER.md §3.2 in the paper's order and notation:
  * workgroup-level tile = C*T consecutive blocks, thread-level tile = T blocks
    (§3.2.1, Fig. 8);
  * strategy 1: each thread runs a sequential segmented scan over its tile into its
    'intermediate_sums' and writes its last partial sum into 'last_partial_sums'
    (0 when its last block is a row stop); start flag = "tile contains a row stop"
    (§3.2.2);
  * parallel (inclusive, segmented) scan of last_partial_sums;
  * combine: the first stop of thread t adds last_partial_sums[t-1] (scanned), and the
    previous workgroup's Grp_sum when the segment spans workgroups (§3.2.3);
  * adjacent synchronization: Grp_sum[X] = last partial sum of X if X holds a row stop,
    else Grp_sum[X-1] + last partial sum of X (§3.2.4);
  * simulate_s2: strategy 2, the per-workgroup result cache addressed by first-result
    entries (§3.2.2, §3.2.3, Figs. 10/12).
Generic over the element type (ints, Fractions, floats): no rounding of its own.
"""
from __future__ import annotations


def simulate(values, bits, T: int, C: int):
    """values[b]: per-block product (already multiplied, step 1 of P:226);
    bits[b]: BCCOO bit flag (0 = row stop).  len must be a multiple of T*C.
    Returns (segment_sums, trace) where trace holds per-workgroup last_partial_sums,
    start flags, the scanned array, and Grp_sum."""
    n = len(values)
    assert n % (T * C) == 0 and len(bits) == n
    zero = values[0] * 0 if n else 0
    results = []
    trace = []
    grp_sum = []
    for X in range(n // (T * C)):
        base = X * T * C
        inter = []           # per-thread intermediate_sums (strategy 1)
        lps = []             # last_partial_sums
        start = []           # start flags
        for t in range(C):
            s = zero
            sums = []
            has_stop = False
            for i in range(T):
                b = base + t * T + i
                s = s + values[b]
                sums.append(s)
                if bits[b] == 0:       # row stop: the sum so far closes a segment
                    has_stop = True
                    s = zero
            inter.append(sums)
            lps.append(s)              # 0 when the last block is a row stop
            start.append(1 if has_stop else 0)
        # parallel segmented (inclusive) scan on last_partial_sums
        scanned = []
        for t in range(C):
            scanned.append(lps[t] if (t == 0 or start[t]) else scanned[t - 1] + lps[t])
        # adjacent synchronization
        if any(start):
            grp = scanned[C - 1]
        else:
            grp = (grp_sum[X - 1] if X > 0 else zero) + scanned[C - 1]
        prev_grp = grp_sum[X - 1] if X > 0 else zero
        grp_sum.append(grp)
        # combine: walk each intermediate_sums array
        for t in range(C):
            first = True
            for i in range(T):
                b = base + t * T + i
                if bits[b] != 0:
                    continue
                v = inter[t][i]
                if first:
                    # segment may span earlier threads of this workgroup ...
                    if t > 0:
                        v = scanned[t - 1] + v
                    # ... and earlier workgroups when no thread before t had a stop
                    if not any(start[:t]):
                        v = prev_grp + v
                    first = False
                # later stops: the running sum restarted after the previous stop, so the
                # intermediate sum is already the complete segment sum
                results.append(v)
        trace.append({"last_partial_sums": lps, "start_flags": start, "scanned": scanned,
                      "grp_sum": grp, "skip_scan": all(start[1:])})
    return results, trace


def simulate_s2(values, bits, T: int, C: int, RC: int):
    """Strategy 2 (§3.2.2, §3.2.3, Figs. 10 and 12), same inputs as
    simulate() plus RC = result cache entries per workgroup (Table 1: a multiple of the
    workgroup size).  Per workgroup, in the paper's order:
      * first-result entries: fre[t] = row stops in the tile before thread t;
      * each thread runs its sequential segmented sum over its tile; at each row stop the
        current sum goes to result-cache entry fre[t] + j (j-th stop of the thread), or to
        the global result array when that entry is >= RC ("larger than the results cache
        size"); its last partial sum goes to last_partial_sums;
      * the parallel segmented scan of last_partial_sums;
      * each thread except thread 0 that has a stop adds last_partial_sums[t-1] (scanned)
        to its first entry; thread 0 adds the previous workgroup's Grp_sum to entry 0 (and
        so does any thread whose first stop is the workgroup's first, i.e. no earlier
        thread of the workgroup had a stop) — the "segments spanning workgroups" case;
      * the cache (and the overflow entries) are the workgroup's segment sums, in order.
    Returns (segment_sums, trace); trace holds per workgroup the cache right after the
    threads' walks ("cache_walk"), after the fix-up ("cache"), and fre."""
    n = len(values)
    assert n % (T * C) == 0 and len(bits) == n and RC >= 1
    zero = values[0] * 0 if n else 0
    results = []
    trace = []
    grp_sum = []
    for X in range(n // (T * C)):
        base = X * T * C
        nst = [sum(1 for i in range(T) if bits[base + t * T + i] == 0) for t in range(C)]
        fre = [sum(nst[:t]) for t in range(C)]
        total = sum(nst)
        cache = [None] * min(RC, total)
        overflow = {}                  # entry -> value, entries >= RC (global result array)
        lps, start = [], []
        for t in range(C):
            s = zero
            j = 0
            for i in range(T):
                b = base + t * T + i
                s = s + values[b]
                if bits[b] == 0:
                    e = fre[t] + j
                    if e < RC:
                        cache[e] = s
                    else:
                        overflow[e] = s
                    j += 1
                    s = zero
            lps.append(s)
            start.append(1 if j else 0)
        cache_walk = list(cache)
        scanned = []
        for t in range(C):
            scanned.append(lps[t] if (t == 0 or start[t]) else scanned[t - 1] + lps[t])
        if any(start):
            grp = scanned[C - 1]
        else:
            grp = (grp_sum[X - 1] if X > 0 else zero) + scanned[C - 1]
        prev_grp = grp_sum[X - 1] if X > 0 else zero
        grp_sum.append(grp)
        for t in range(C):
            if not start[t]:
                continue
            e = fre[t]
            v = cache[e] if e < RC else overflow[e]
            if t > 0:
                v = scanned[t - 1] + v
            if not any(start[:t]):
                v = prev_grp + v
            if e < RC:
                cache[e] = v
            else:
                overflow[e] = v
        results.extend(cache[e] if e < RC else overflow[e] for e in range(total))
        trace.append({"fre": fre, "cache_walk": cache_walk, "cache": list(cache), "last_partial_sums": lps,
                      "scanned": scanned, "grp_sum": grp})
    return results, trace
