"""Oracle: deterministic placement simulator and canonical trace.

Paper anchors: work "divided equally across number of processes" (PAPER.md
Fig. 4 caption, §5.2) -> STATIC (k-1) mod P, done by the caller with
explicit partitions (A6); a GPU listed several times with a GPU% each (P:173,
§4.1) -> several partitions per GPU; MIG fixed slices (§4.2) and the
equal/fill layouts. MPS GPU% is an SM budget; here budgets
are whole 8-SM groups of one driver split (green-context granularity, A20).

Rules written out (the C++ runtime implements the same rules independently):
  * groups: k = ceil(sm/group_size) lowest-index free groups; a request of
    >= total_sms (or k > n_groups) is the WHOLE device (all groups + the
    remainder SMs, sm_count = total_sms) and needs every group free.
  * resize: the partition's own groups are released first, then reallocated
    lowest-first by the same rule (restored on failure, MX_ENOSM).
  * I5: sum of live quotas on a GPU <= device memory, else MX_ENOMEM.
  * ANY = weighted least-assigned-work: argmin_p (A_p + c_k)/s_p compared
    exactly as (A_p + c_k)*s_q < (A_q + c_k)*s_p, ties -> lowest part id;
    then A_p += c_k. A_p is never decremented (timing-independent). Explicit
    placements add c_k to A_p as well.
  * trace: little-endian records of 8 x u64; timestamps excluded. CREATE /
    RESIZE carry a flag word (bit0 whole device, bit1 shared = unpartitioned).
  * shared partitions (N1) own no groups and do not count toward I2.
"""
from __future__ import annotations

import hashlib
import struct
from dataclasses import dataclass, field

MX_OK, MX_ENODEV, MX_EINVAL, MX_ENOSM, MX_ENOMEM = 0, -19, -22, -28, -12
MX_PART_ANY = -1

REC_HEADER, REC_CREATE, REC_RESIZE, REC_DESTROY, REC_PLACE = 0, 1, 2, 3, 4
TRACE_VERSION = 1


class SchedError(Exception):
    def __init__(self, code):
        super().__init__(code)
        self.code = code


@dataclass
class Part:
    pid: int
    gpu: int
    groups: list
    sm_count: int
    whole: bool
    quota: int
    epoch: int = 0
    live: bool = True
    assigned: int = 0
    seq: int = 0
    shared: bool = False

    @property
    def mask(self) -> int:
        m = 0
        for g in self.groups:
            m |= 1 << g
        return m


@dataclass
class Sim:
    n_gpus: int
    n_groups: int = 18
    group_size: int = 8
    total_sms: int = 148
    mem_bytes: int = 180 * 10 ** 9
    parts: list = field(default_factory=list)
    records: list = field(default_factory=list)
    placements: list = field(default_factory=list)
    next_task: int = 1

    def __post_init__(self):
        self.records.append((REC_HEADER, TRACE_VERSION, self.n_gpus, self.n_groups,
                             self.group_size, self.total_sms, 0, 0))

    # -- groups ---------------------------------------------------------------
    def _free_groups(self, gpu: int, exclude: int | None = None) -> list:
        used = set()
        for p in self.parts:
            if p.live and p.gpu == gpu and p.pid != exclude:
                used.update(p.groups)
        return [g for g in range(self.n_groups) if g not in used]

    def _alloc(self, gpu: int, sm: int, exclude=None):
        free = self._free_groups(gpu, exclude)
        k = -(-sm // self.group_size)
        if sm >= self.total_sms or k > self.n_groups:
            if len(free) != self.n_groups:
                raise SchedError(MX_ENOSM)
            return list(range(self.n_groups)), self.total_sms, True
        if len(free) < k:
            raise SchedError(MX_ENOSM)
        return free[:k], k * self.group_size, False

    def _quota_ok(self, gpu: int, quota: int, exclude=None) -> bool:
        s = sum(p.quota for p in self.parts if p.live and p.gpu == gpu and p.pid != exclude)
        return s + quota <= self.mem_bytes

    # -- events ---------------------------------------------------------------
    def create(self, gpu: int, sm: int, hbm: int) -> int:
        if gpu < 0 or gpu >= self.n_gpus:
            raise SchedError(MX_ENODEV)
        if sm <= 0 or hbm <= 0:
            raise SchedError(MX_EINVAL)
        if not self._quota_ok(gpu, hbm):
            raise SchedError(MX_ENOMEM)
        groups, smc, whole = self._alloc(gpu, sm)
        p = Part(len(self.parts), gpu, groups, smc, whole, hbm)
        self.parts.append(p)
        self.records.append((REC_CREATE, p.pid, gpu, smc, p.mask, hbm, 0, int(whole)))
        return p.pid

    def create_shared(self, gpu: int, n_ctas: int, hbm: int) -> int:
        """Unpartitioned stream on the whole device (the
        time-sharing / default-MPS comparison modes of PAPER.md Table 1):
        owns no SM groups, sm_count = min(n_ctas, total_sms) is its grid and WLAW weight."""
        if gpu < 0 or gpu >= self.n_gpus:
            raise SchedError(MX_ENODEV)
        if n_ctas <= 0 or hbm <= 0:
            raise SchedError(MX_EINVAL)
        if not self._quota_ok(gpu, hbm):
            raise SchedError(MX_ENOMEM)
        p = Part(len(self.parts), gpu, [], min(n_ctas, self.total_sms), False, hbm, shared=True)
        self.parts.append(p)
        self.records.append((REC_CREATE, p.pid, gpu, p.sm_count, 0, hbm, 0, 2))
        return p.pid

    def _flags(self, p: Part) -> int:
        return int(p.whole) | (2 if p.shared else 0)

    def _live(self, pid: int) -> Part:
        if pid < 0 or pid >= len(self.parts) or not self.parts[pid].live:
            raise SchedError(MX_EINVAL)
        return self.parts[pid]

    def resize(self, pid: int, sm: int, hbm: int):
        p = self._live(pid)
        sm = p.sm_count if sm <= 0 else sm
        hbm = p.quota if hbm == 0 else hbm
        if not self._quota_ok(p.gpu, hbm, exclude=pid):
            raise SchedError(MX_ENOMEM)
        if p.shared:
            groups, smc, whole = [], min(sm, self.total_sms), False
        else:
            groups, smc, whole = self._alloc(p.gpu, sm, exclude=pid)
        p.groups, p.sm_count, p.whole, p.quota = groups, smc, whole, hbm
        p.epoch += 1
        self.records.append((REC_RESIZE, pid, p.gpu, smc, p.mask, hbm, p.epoch, self._flags(p)))

    def destroy(self, pid: int):
        p = self._live(pid)
        p.live = False
        self.records.append((REC_DESTROY, pid, p.gpu, 0, 0, 0, p.epoch, 0))

    def submit(self, fn: int, part: int, cost: int) -> tuple:
        if part == MX_PART_ANY:
            live = [p for p in self.parts if p.live]
            if not live:
                raise SchedError(MX_EINVAL)
            best = live[0]
            for q in live[1:]:
                # q better than best iff (A_q + c)/s_q < (A_best + c)/s_best
                if (q.assigned + cost) * best.sm_count < (best.assigned + cost) * q.sm_count:
                    best = q
            p = best
        else:
            p = self._live(part)
        tid = self.next_task
        self.next_task += 1
        seq = p.seq
        p.seq += 1
        p.assigned += cost
        self.records.append((REC_PLACE, tid, fn, p.gpu, p.pid, seq, p.epoch, cost))
        self.placements.append((tid, fn, p.gpu, p.pid, seq, p.epoch, cost))
        return tid, p.pid, seq

    # -- serialisation --------------------------------------------------------
    def trace_bytes(self) -> bytes:
        return b"".join(struct.pack("<8Q", *[int(v) & (2 ** 64 - 1) for v in r])
                        for r in self.records)

    def trace_sha256(self) -> str:
        return hashlib.sha256(self.trace_bytes()).hexdigest()


def parse_trace(data: bytes) -> list:
    assert len(data) % 64 == 0
    return [struct.unpack_from("<8Q", data, i) for i in range(0, len(data), 64)]


def static_part(task_id: int, n_parts: int) -> int:
    """STATIC placement of P:195 ('divided equally'), reading A6: (k-1) mod P."""
    return (task_id - 1) % n_parts
