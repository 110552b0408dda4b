"""Oracle: run invariants I1-I6, checked on GPU traces.

BASELINE.json north_star: "every task completes exactly once, partition SM
budgets sum to at most 148, and no partition exceeds its HBM quota". The paper
anchors: per-process partitions with SM budgets (§4.1) and MIG memory
isolation (Table 1; A23 — here an allocator quota, not hardware).
Each checker returns a list of violation strings (empty = holds).
"""
from __future__ import annotations

from collections import defaultdict

from .sched import REC_CREATE, REC_RESIZE, REC_DESTROY, REC_PLACE


def i1_exactly_once(submitted_ids, results) -> list:
    """I1: every submitted task id has exactly one completion with a status."""
    seen = defaultdict(int)
    for r in results:
        seen[r["task"]] += 1
    errs = [f"task {t} completed {seen[t]} times" for t in submitted_ids if seen[t] != 1]
    errs += [f"unknown task {t} completed" for t in seen if t not in set(submitted_ids)]
    return errs


def i2_sm_budget(records, total_sms: int = 148) -> list:
    """I2: per GPU after every CREATE/RESIZE, sum sm_count <= total and groups disjoint."""
    errs = []
    live = {}
    for r in records:
        typ = r[0]
        if typ in (REC_CREATE, REC_RESIZE):
            if r[7] & 2:            # shared (unpartitioned) stream: owns no SMs
                live.pop(r[1], None)
                continue
            live[r[1]] = (r[2], r[3], r[4])
        elif typ == REC_DESTROY:
            live.pop(r[1], None)
        else:
            continue
        by_gpu = defaultdict(list)
        for pid, (gpu, sm, mask) in live.items():
            by_gpu[gpu].append((pid, sm, mask))
        for gpu, ps in by_gpu.items():
            if sum(sm for _, sm, _ in ps) > total_sms:
                errs.append(f"gpu {gpu}: SM budget {sum(sm for _, sm, _ in ps)} > {total_sms}")
            acc = 0
            for pid, _, mask in ps:
                if acc & mask:
                    errs.append(f"gpu {gpu}: part {pid} overlaps groups")
                acc |= mask
    return errs


def i3_quota(part_infos) -> list:
    """I3: per partition hbm_peak <= quota (part_query snapshots)."""
    return [f"part {i['part']}: peak {i['hbm_peak']} > quota {i['hbm_quota']}"
            for i in part_infos if i["hbm_peak"] > i["hbm_quota"]]


def i4_fifo(results) -> list:
    """I4: per partition, completions (t_end) are monotone in seq_in_part."""
    errs = []
    by_part = defaultdict(list)
    for r in results:
        by_part[r["part"]].append((r["seq"], r["t_end"], r["task"]))
    for p, lst in by_part.items():
        lst.sort()
        for a, b in zip(lst, lst[1:]):
            if b[1] < a[1]:
                errs.append(f"part {p}: task {b[2]} (seq {b[0]}) ended before seq {a[0]}")
    return errs


def i5_quota_sum(records, mem_bytes: int) -> list:
    """I5: sum of quotas per GPU <= device memory after every CREATE/RESIZE."""
    errs = []
    live = {}
    for r in records:
        if r[0] in (REC_CREATE, REC_RESIZE):
            live[r[1]] = (r[2], r[5])
        elif r[0] == REC_DESTROY:
            live.pop(r[1], None)
        else:
            continue
        tot = defaultdict(int)
        for gpu, q in live.values():
            tot[gpu] += q
        errs += [f"gpu {g}: quotas {q} > mem {mem_bytes}" for g, q in tot.items() if q > mem_bytes]
    return errs


def i6_smid_subset(observed_smids: set, allowed_smids: set, sm_count: int) -> list:
    """I6: the %smid set observed for a partition has at most sm_count SMs and,
    where the SM ids of the partition are known, lies inside them."""
    errs = []
    if len(observed_smids) > sm_count:
        errs.append(f"observed {len(observed_smids)} SMs > budget {sm_count}")
    if allowed_smids and not observed_smids <= allowed_smids:
        errs.append(f"SMs outside partition: {sorted(observed_smids - allowed_smids)}")
    return errs


def placements_from_trace(records) -> list:
    return [r[1:] for r in records if r[0] == REC_PLACE]
