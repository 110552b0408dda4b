"""Thin ctypes binding of include/mx.h (argument marshalling only).

Every step of the hot path runs in libmx.so (CUDA kernels for sm_100a + the
C++ runtime). There is no Python or CPU fallback: if the library is missing
the import raises, and without a CC 10.x GPU `mx_init` fails with MX_ENODEV.
Names follow the C ABI (part_create, fn_register, fn_submit, fn_wait,
part_resize, ...); see include/mx.h for semantics and PAPER.md citations.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MX_LIB") or os.path.join(_HERE, "libmx.so")

MX_OK, MX_ENOENT, MX_EDEVICE, MX_ENOMEM, MX_EBUSY = 0, -2, -5, -12, -16
MX_ENODEV, MX_EINVAL, MX_ENOSM, MX_ETIMEDOUT, MX_ESTATE = -19, -22, -28, -110, -125
MX_PART_ANY = -1
MX_FN_DECODE, MX_FN_MPNN, MX_FN_MPNN_TRAIN = 1, 2, 3
MX_FN_SHARED_WEIGHTS = 1


class MxError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"{what}: {code} ({strerror(code)}) {last_error()}")
        self.code = code


class DecodeCfgC(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("d_model", C.c_int32), ("n_heads", C.c_int32),
                ("n_kv_heads", C.c_int32), ("head_dim", C.c_int32), ("d_ff", C.c_int32),
                ("vocab", C.c_int32), ("max_seq", C.c_int32), ("max_batch", C.c_int32),
                ("rms_eps", C.c_float), ("rope_theta", C.c_float)]


class MpnnCfgC(C.Structure):
    _fields_ = [("n_atom_types", C.c_int32), ("n_bond_types", C.c_int32), ("hidden", C.c_int32),
                ("steps", C.c_int32), ("max_mols", C.c_int32), ("max_atoms", C.c_int32),
                ("max_edges", C.c_int32)]


class FnDescC(C.Structure):
    _fields_ = [("kind", C.c_int32), ("flags", C.c_uint32), ("weight_seed", C.c_uint64),
                ("dec", DecodeCfgC), ("mpnn", MpnnCfgC)]


class TaskDescC(C.Structure):
    _fields_ = [("fn", C.c_int32), ("batch", C.c_int32), ("prompt_len", C.c_int32),
                ("gen_len", C.c_int32), ("prompt", C.c_void_p), ("out_tokens", C.c_void_p),
                ("out_logits", C.c_void_p), ("n_mol", C.c_int32), ("n_atoms", C.c_int32),
                ("n_edges", C.c_int32), ("reserved", C.c_int32), ("atom_off", C.c_void_p),
                ("atom_type", C.c_void_p), ("edge_off", C.c_void_p), ("edges", C.c_void_p),
                ("out_ip", C.c_void_p), ("cost", C.c_uint64), ("targets", C.c_void_p),
                ("out_loss", C.c_void_p), ("lr", C.c_float), ("reserved2", C.c_int32)]


class ResultC(C.Structure):
    _fields_ = [("status", C.c_int32), ("gpu", C.c_int32), ("part", C.c_int32),
                ("epoch", C.c_uint32), ("seq_in_part", C.c_uint64), ("t_submit_ns", C.c_uint64),
                ("t_start_ns", C.c_uint64), ("t_end_ns", C.c_uint64), ("kernel_ns", C.c_uint64)]


class PartInfoC(C.Structure):
    _fields_ = [("gpu", C.c_int32), ("sm_count", C.c_int32), ("n_ctas", C.c_int32),
                ("whole", C.c_int32), ("group_mask", C.c_uint64), ("hbm_quota", C.c_uint64),
                ("hbm_used", C.c_uint64), ("hbm_peak", C.c_uint64), ("epoch", C.c_uint32),
                ("shared", C.c_uint32)]


class GpuInfoC(C.Structure):
    _fields_ = [("ordinal", C.c_int32), ("sm_total", C.c_int32), ("n_groups", C.c_int32),
                ("group_size", C.c_int32), ("remainder_sms", C.c_int32), ("cc_major", C.c_int32),
                ("cc_minor", C.c_int32), ("reserved", C.c_int32), ("mem_bytes", C.c_uint64)]


# symbol -> (restype, argtypes)
_SIGS = {
    "mx_init": (C.c_int32, [C.c_uint32]),
    "mx_init_devices": (C.c_int32, [C.POINTER(C.c_int32), C.c_int32, C.c_uint32]),
    "mx_shutdown": (C.c_int32, []),
    "mx_gpu_count": (C.c_int32, [C.POINTER(C.c_int32)]),
    "mx_gpu_query": (C.c_int32, [C.c_int32, C.POINTER(GpuInfoC)]),
    "mx_strerror": (C.c_char_p, [C.c_int32]),
    "mx_last_error": (C.c_char_p, []),
    "part_create": (C.c_int32, [C.c_int32, C.c_int32, C.c_uint64, C.POINTER(C.c_int32)]),
    "part_create_shared": (C.c_int32, [C.c_int32, C.c_int32, C.c_uint64, C.POINTER(C.c_int32)]),
    "part_resize": (C.c_int32, [C.c_int32, C.c_int32, C.c_uint64]),
    "part_destroy": (C.c_int32, [C.c_int32]),
    "part_query": (C.c_int32, [C.c_int32, C.POINTER(PartInfoC)]),
    "fn_register": (C.c_int32, [C.POINTER(FnDescC), C.POINTER(C.c_int32)]),
    "fn_load": (C.c_int32, [C.c_int32, C.c_int32]),
    "mx_weight_pool_query": (C.c_int32, [C.c_int32, C.POINTER(C.c_uint64), C.POINTER(C.c_int32)]),
    "fn_submit": (C.c_int32, [C.c_int32, C.POINTER(TaskDescC), C.POINTER(C.c_uint64)]),
    "fn_wait": (C.c_int32, [C.c_uint64, C.c_int64, C.POINTER(ResultC)]),
    "mx_task_default_cost": (C.c_int32, [C.POINTER(FnDescC), C.POINTER(TaskDescC),
                                         C.POINTER(C.c_uint64)]),
    "mx_trace_write": (C.c_int32, [C.c_char_p]),
    "fn_read_tensor": (C.c_int32, [C.c_int32, C.c_int32, C.c_int32, C.c_void_p, C.c_uint64]),
    "mx_probe_smids": (C.c_int32, [C.c_int32, C.c_int32, C.c_uint64, C.POINTER(C.c_uint32)]),
    "mx_probe_smids_concurrent": (C.c_int32, [C.POINTER(C.c_int32), C.c_int32, C.c_int32,
                                              C.c_uint64, C.POINTER(C.c_uint32)]),
    "mx_launch_count": (C.c_int32, [C.POINTER(C.c_uint64)]),
    "mx_debug_inject_error": (C.c_int32, [C.c_int32, C.c_int32]),
    "mx_decode_profile": (C.c_int32, [C.c_int32, C.POINTER(C.c_uint64), C.c_int32]),
    "mx_sched_new": (C.c_void_p, [C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_uint64]),
    "mx_sched_free": (None, [C.c_void_p]),
    "mx_sched_create": (C.c_int32, [C.c_void_p, C.c_int32, C.c_int32, C.c_uint64,
                                    C.POINTER(C.c_int32)]),
    "mx_sched_create_shared": (C.c_int32, [C.c_void_p, C.c_int32, C.c_int32, C.c_uint64,
                                           C.POINTER(C.c_int32)]),
    "mx_sched_resize": (C.c_int32, [C.c_void_p, C.c_int32, C.c_int32, C.c_uint64]),
    "mx_sched_destroy": (C.c_int32, [C.c_void_p, C.c_int32]),
    "mx_sched_submit": (C.c_int32, [C.c_void_p, C.c_int32, C.c_int32, C.c_uint64,
                                    C.POINTER(C.c_uint64), C.POINTER(C.c_int32),
                                    C.POINTER(C.c_uint64)]),
    "mx_rightsize": (C.c_int32, [C.POINTER(C.c_int32), C.POINTER(C.c_double), C.c_int32, C.c_int32,
                                 C.c_int32, C.c_int32, C.c_double, C.POINTER(C.c_int32),
                                 C.POINTER(C.c_int32), C.POINTER(C.c_double)]),
    "mx_sched_trace": (C.c_int32, [C.c_void_p, C.c_void_p, C.c_uint64, C.POINTER(C.c_uint64)]),
    "fn_rightsize": (C.c_int32, [C.c_int32, C.c_int32, C.POINTER(TaskDescC), C.c_uint64,
                                 C.POINTER(C.c_int32), C.c_int32, C.c_int32, C.c_int32, C.c_double,
                                 C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_double),
                                 C.POINTER(C.c_double)]),
}

_lib = None


def lib() -> C.CDLL:
    """Load libmx.so (fails loudly if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_sc_dhakalrwercfm23_b200.build`")
        os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def strerror(code: int) -> str:
    return lib().mx_strerror(code).decode()


def last_error() -> str:
    return lib().mx_last_error().decode()


def _check(code: int, what: str):
    if code != MX_OK:
        raise MxError(code, what)


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


# ---------------------------------------------------------------------------
# Lifecycle and partitions
# ---------------------------------------------------------------------------

def mx_init(devices=None, flags: int = 0):
    if devices is None:
        _check(lib().mx_init(flags), "mx_init")
    else:
        arr = (C.c_int32 * len(devices))(*devices)
        _check(lib().mx_init_devices(arr, len(devices), flags), "mx_init_devices")


def mx_shutdown():
    _check(lib().mx_shutdown(), "mx_shutdown")


def mx_gpu_count() -> int:
    n = C.c_int32()
    _check(lib().mx_gpu_count(C.byref(n)), "mx_gpu_count")
    return n.value


def mx_gpu_query(gpu: int) -> dict:
    g = GpuInfoC()
    _check(lib().mx_gpu_query(gpu, C.byref(g)), "mx_gpu_query")
    return {k: getattr(g, k) for k, _ in GpuInfoC._fields_}


def part_create(gpu: int, sm_count: int, hbm_bytes: int) -> int:
    p = C.c_int32()
    _check(lib().part_create(gpu, sm_count, hbm_bytes, C.byref(p)), "part_create")
    return p.value


def part_create_shared(gpu: int, n_ctas: int, hbm_bytes: int) -> int:
    """Unpartitioned stream (N1 comparison modes): no SM groups, grid = n_ctas."""
    p = C.c_int32()
    _check(lib().part_create_shared(gpu, n_ctas, hbm_bytes, C.byref(p)), "part_create_shared")
    return p.value


def part_resize(part: int, sm_count: int = 0, hbm_bytes: int = 0):
    _check(lib().part_resize(part, sm_count, hbm_bytes), "part_resize")


def part_destroy(part: int):
    _check(lib().part_destroy(part), "part_destroy")


def part_query(part: int) -> dict:
    i = PartInfoC()
    _check(lib().part_query(part, C.byref(i)), "part_query")
    return {k: getattr(i, k) for k, _ in PartInfoC._fields_}


# ---------------------------------------------------------------------------
# Functions and tasks
# ---------------------------------------------------------------------------

def decode_desc(cfg, max_batch: int = 1, seed: int | None = None,
                shared_weights: bool = False) -> FnDescC:
    d = FnDescC()
    d.kind = MX_FN_DECODE
    d.flags = MX_FN_SHARED_WEIGHTS if shared_weights else 0
    d.weight_seed = cfg.seed if seed is None else seed
    d.dec = DecodeCfgC(cfg.n_layers, cfg.d_model, cfg.n_heads, cfg.n_kv_heads, cfg.head_dim,
                       cfg.d_ff, cfg.vocab, cfg.max_seq, max_batch, cfg.rms_eps, cfg.rope_theta)
    return d


def mpnn_desc(cfg, max_mols: int, max_atoms: int, max_edges: int,
              shared_weights: bool = False) -> FnDescC:
    d = FnDescC()
    d.kind = MX_FN_MPNN
    d.flags = MX_FN_SHARED_WEIGHTS if shared_weights else 0
    d.weight_seed = cfg.seed
    d.mpnn = MpnnCfgC(cfg.n_atom_types, cfg.n_bond_types, cfg.hidden, cfg.steps, max_mols,
                      max_atoms, max_edges)
    return d


def fn_register(desc: FnDescC) -> int:
    f = C.c_int32()
    _check(lib().fn_register(C.byref(desc), C.byref(f)), "fn_register")
    return f.value


def weight_pool_query(gpu: int) -> dict:
    """Shared read-only weight pool of `gpu` (N3): bytes used and functions held."""
    used, n = C.c_uint64(0), C.c_int32(0)
    _check(lib().mx_weight_pool_query(gpu, C.byref(used), C.byref(n)), "mx_weight_pool_query")
    return {"used_bytes": used.value, "n_fns": n.value}


def fn_load(fn: int, part: int):
    _check(lib().fn_load(fn, part), "fn_load")


class Task:
    """Owns the numpy input/output buffers of one submitted task until fn_wait."""

    def __init__(self, fn: int):
        self.fn = fn
        self.desc = TaskDescC()
        self.desc.fn = fn
        self.keep = []
        self.id = 0
        self.tokens = self.logits = self.ip = self.loss = None


def decode_task(fn: int, prompt: np.ndarray, gen_len: int, want_logits: bool = False,
                vocab: int = 0, cost: int = 0) -> Task:
    prompt = np.ascontiguousarray(prompt, dtype=np.int32)
    B, P = prompt.shape
    t = Task(fn)
    t.tokens = np.zeros((B, gen_len), dtype=np.int32)
    if want_logits:
        t.logits = np.zeros((gen_len, B, vocab), dtype=np.float32)
    d = t.desc
    d.batch, d.prompt_len, d.gen_len = B, P, gen_len
    d.prompt, d.out_tokens, d.out_logits = _ptr(prompt), _ptr(t.tokens), _ptr(t.logits)
    d.cost = cost
    t.keep = [prompt]
    return t


def mpnn_task(fn: int, mol: dict, cost: int = 0) -> Task:
    """mol = workloads.inputs.molecules(...) (CSR arrays)."""
    ao = np.ascontiguousarray(mol["atom_off"], dtype=np.int32)
    at = np.ascontiguousarray(mol["atom_type"], dtype=np.uint8)
    eo = np.ascontiguousarray(mol["edge_off"], dtype=np.int32)
    ed = np.ascontiguousarray(mol["edges"])
    assert ed.dtype.itemsize == 6
    t = Task(fn)
    M = len(ao) - 1
    t.ip = np.zeros(M, dtype=np.float32)
    d = t.desc
    d.n_mol, d.n_atoms, d.n_edges = M, len(at), len(ed)
    d.atom_off, d.atom_type, d.edge_off = _ptr(ao), _ptr(at), _ptr(eo)
    d.edges = _ptr(ed) if len(ed) else None
    d.out_ip = _ptr(t.ip)
    d.cost = cost
    t.keep = [ao, at, eo, ed]
    return t


def mpnn_train_desc(cfg, max_mols: int, max_atoms: int, max_edges: int) -> FnDescC:
    """IP-emulator training step function (N4): fp32 parameters per instance."""
    d = mpnn_desc(cfg, max_mols, max_atoms, max_edges)
    d.kind = MX_FN_MPNN_TRAIN
    return d


def mpnn_train_task(fn: int, mol: dict, targets: np.ndarray, lr: float, cost: int = 0) -> Task:
    """One SGD step on the molecules `mol` with `targets`; after fn_wait,
    task.ip = predictions before the update, task.loss[0] = the loss."""
    t = mpnn_task(fn, mol, cost)
    tg = np.ascontiguousarray(targets, dtype=np.float32)
    assert tg.shape == t.ip.shape
    t.loss = np.zeros(1, dtype=np.float32)
    t.desc.targets, t.desc.out_loss, t.desc.lr = _ptr(tg), _ptr(t.loss), float(lr)
    t.keep.append(tg)
    return t


def fn_read_params(fn: int, part: int, tensor_id: int, n_elems: int) -> np.ndarray:
    """fp32 training state of a MX_FN_MPNN_TRAIN instance (tensor ids as C1)."""
    out = np.empty(n_elems, dtype=np.float32)
    _check(lib().fn_read_tensor(fn, part, tensor_id, _ptr(out), n_elems * 4), "fn_read_tensor")
    return out


def fn_submit(part: int, task: Task) -> int:
    tid = C.c_uint64()
    _check(lib().fn_submit(part, C.byref(task.desc), C.byref(tid)), "fn_submit")
    task.id = tid.value
    return task.id


def fn_wait(task, timeout_ns: int = -1) -> dict:
    tid = task.id if isinstance(task, Task) else int(task)
    r = ResultC()
    _check(lib().fn_wait(tid, timeout_ns, C.byref(r)), "fn_wait")
    return {"task": tid, **{k: getattr(r, k) for k, _ in ResultC._fields_}}


def task_default_cost(desc: FnDescC, task: Task) -> int:
    c = C.c_uint64()
    _check(lib().mx_task_default_cost(C.byref(desc), C.byref(task.desc), C.byref(c)),
           "mx_task_default_cost")
    return c.value


def mx_trace_write(path: str):
    _check(lib().mx_trace_write(path.encode()), "mx_trace_write")


def fn_read_tensor(fn: int, part: int, tensor_id: int, n_elems: int) -> np.ndarray:
    out = np.empty(n_elems, dtype=np.uint16)
    _check(lib().fn_read_tensor(fn, part, tensor_id, _ptr(out), n_elems * 2), "fn_read_tensor")
    return out


def probe_smids(part: int, n_ctas: int, spin_ns: int = 200_000) -> np.ndarray:
    out = np.zeros(n_ctas, dtype=np.uint32)
    _check(lib().mx_probe_smids(part, n_ctas, spin_ns, out.ctypes.data_as(C.POINTER(C.c_uint32))),
           "mx_probe_smids")
    return out


def probe_smids_concurrent(parts, n_ctas: int, spin_ns: int = 2_000_000) -> np.ndarray:
    arr = (C.c_int32 * len(parts))(*parts)
    out = np.zeros(len(parts) * n_ctas, dtype=np.uint32)
    _check(lib().mx_probe_smids_concurrent(arr, len(parts), n_ctas, spin_ns,
                                           out.ctypes.data_as(C.POINTER(C.c_uint32))),
           "mx_probe_smids_concurrent")
    return out.reshape(len(parts), n_ctas)


def decode_profile(part: int, n_ctas: int) -> np.ndarray:
    out = np.zeros(n_ctas * 8, dtype=np.uint64)
    _check(lib().mx_decode_profile(part, out.ctypes.data_as(C.POINTER(C.c_uint64)), n_ctas * 8),
           "mx_decode_profile")
    return out.reshape(n_ctas, 8)


def debug_inject_error(part: int, code: int = 7):
    """Fault-path test hook: the next task launched on `part` reports device error `code`."""
    _check(lib().mx_debug_inject_error(part, code), "mx_debug_inject_error")


def launch_count() -> int:
    c = C.c_uint64()
    _check(lib().mx_launch_count(C.byref(c)), "mx_launch_count")
    return c.value


def rightsize(sms, t, total_sms=148, max_parts=37, objective=1, slack=0.0):
    """N2 right-sizing (mx_rightsize): -> (sm_per_partition, n_partitions, predicted rate)."""
    n = len(sms)
    a = (C.c_int32 * n)(*[int(x) for x in sms])
    b = (C.c_double * n)(*[float(x) for x in t])
    o_sm, o_p, o_r = C.c_int32(), C.c_int32(), C.c_double()
    _check(lib().mx_rightsize(a, b, n, total_sms, max_parts, objective, slack, C.byref(o_sm),
                              C.byref(o_p), C.byref(o_r)), "mx_rightsize")
    return o_sm.value, o_p.value, o_r.value


def fn_rightsize(fn: int, gpu: int, sample: Task, cand_sms, hbm_bytes: int = 1 << 30,
                 reps: int = 2, objective: int = 1, slack: float = 0.0):
    """N2: measure `sample` alone on each candidate partition size, then right-size.
    -> dict(sm, parts, rate_per_s, curve=[(sms, t_ns)])"""
    n = len(cand_sms)
    a = (C.c_int32 * n)(*[int(x) for x in cand_sms])
    tt = (C.c_double * n)(*([0.0] * n))
    o_sm, o_p, o_r = C.c_int32(), C.c_int32(), C.c_double()
    _check(lib().fn_rightsize(fn, gpu, C.byref(sample.desc), hbm_bytes, a, n, reps, objective, slack,
                              C.byref(o_sm), C.byref(o_p), C.byref(o_r), tt), "fn_rightsize")
    return {"sm": o_sm.value, "parts": o_p.value, "rate_per_s": o_r.value * 1e9,
            "curve": [(int(cand_sms[i]), float(tt[i])) for i in range(n) if tt[i] > 0]}


# ---------------------------------------------------------------------------
# Host-only placement engine (same C++ object the runtime uses)
# ---------------------------------------------------------------------------

class HostSched:
    def __init__(self, n_gpus=1, n_groups=18, group_size=8, total_sms=148, mem_bytes=180 * 10 ** 9):
        self.h = lib().mx_sched_new(n_gpus, n_groups, group_size, total_sms, mem_bytes)
        if not self.h:
            raise MxError(MX_EINVAL, "mx_sched_new")

    def __del__(self):
        if getattr(self, "h", None):
            lib().mx_sched_free(self.h)
            self.h = None

    def create(self, gpu, sm, hbm) -> int:
        p = C.c_int32()
        _check(lib().mx_sched_create(self.h, gpu, sm, hbm, C.byref(p)), "mx_sched_create")
        return p.value

    def create_shared(self, gpu, n_ctas, hbm) -> int:
        p = C.c_int32()
        _check(lib().mx_sched_create_shared(self.h, gpu, n_ctas, hbm, C.byref(p)),
               "mx_sched_create_shared")
        return p.value

    def resize(self, part, sm, hbm):
        _check(lib().mx_sched_resize(self.h, part, sm, hbm), "mx_sched_resize")

    def destroy(self, part):
        _check(lib().mx_sched_destroy(self.h, part), "mx_sched_destroy")

    def submit(self, fn, part, cost):
        t, p, s = C.c_uint64(), C.c_int32(), C.c_uint64()
        _check(lib().mx_sched_submit(self.h, fn, part, cost, C.byref(t), C.byref(p), C.byref(s)),
               "mx_sched_submit")
        return t.value, p.value, s.value

    def trace_bytes(self) -> bytes:
        n = C.c_uint64()
        lib().mx_sched_trace(self.h, None, 0, C.byref(n))
        buf = C.create_string_buffer(n.value)
        lib().mx_sched_trace(self.h, buf, n.value, C.byref(n))
        return buf.raw[: n.value]
