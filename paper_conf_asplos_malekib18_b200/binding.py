"""ctypes binding of libplr_b200.so (include/plr.h).  Marshalling only."""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PLR_LIB") or os.path.join(_HERE, "libplr_b200.so")   # PLR_LIB: experiment variants
PAYLOAD_BYTES = 64

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libplr_b200.so is not built (run `python -c 'import __graft_entry__ as g; g.build()'` or "
        "`python paper_conf_asplos_malekib18_b200/build.py`); there is no fallback path")

lib = ctypes.CDLL(LIB_PATH)

_P = ctypes.c_void_p
_S = ctypes.c_size_t
_I = ctypes.c_int
_st = ctypes.c_int

_SIGS = {
    "plr_plan_create": ([ctypes.POINTER(_P), _P, _I, _P, _I, _I, _S], _st),
    "plr_plan_create_cascade": ([ctypes.POINTER(_P), _I, _P, _P, _P, _P, _I, _S], _st),
    "plr_plan_get_signature": ([_P, _P, _P], _st),
    "plr_plan_destroy": ([_P], _st),
    "plr_plan_get_info": ([_P, _P], _st),
    "plr_plan_factor_lists": ([_P, ctypes.c_int64, _P], _st),
    "plr_plan_debug_stats": ([_P, _P, _I], _st),
    "plr_execute": ([_P, _P, _P, _S, _P], _st),
    "plr_execute_continue": ([_P, _P, _P, _S, _P, _P, _P], _st),
    "plr_execute_reverse": ([_P, _P, _P, _S, _P], _st),
    "plr_scan_comparator": ([_P, _P, _P, _S, _P], _st),
    "plr_execute_bidirectional": ([_P, _P, _P, _S, _P, _P], _st),
    "plr_reduce": ([_P, _P, _S, _P, _P], _st),
    "plr_payload_from_output": ([_P, _P, _P, _S, _P, _P], _st),
    "plr_combine": ([_P, _P, _I, _I, _P, _P], _st),
    "plr_combine_host": ([_P, _P, _I, _I, _P], _st),
    "plr_fixup": ([_P, _P, _S, _P, _P], _st),
    "plr_execute_sharded": ([_P, _P, _P, _S, _I, _I, _P, _P], _st),
    "plr_execute_host": ([_P, _P, _P, _S, _P], _st),
    "plr_nccl_unique_id": ([_P, _S], _st),
    "plr_nccl_comm_init": ([ctypes.POINTER(_P), _P, _I, _I], _st),
    "plr_nccl_comm_destroy": ([_P], _st),
    "plr_status_string": ([_I], ctypes.c_char_p),
    "plr_last_error": ([], ctypes.c_char_p),
    "plr_abi_version": ([], _I),
}
for _name, (_args, _res) in _SIGS.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = _res

EXPORTED = tuple(_SIGS)

_DTYPES = {"int32": 0, "float32": 1}
_CLASSES = {0: "ONES", 1: "PERM", 2: "POLY", 3: "DECAY", 4: "FLOAT"}


class PlanInfo(ctypes.Structure):
    _fields_ = [("p", _I), ("k", _I), ("dtype", _I), ("cls", _I), ("elems_per_thread", _I),
                ("threads_per_cta", _I), ("tile_elems", _I), ("stages", _I), ("decay_len", ctypes.c_int64),
                ("fixup_len", ctypes.c_int64), ("n_max", _S), ("scratch_bytes", _S), ("ctas_per_sm", _I),
                ("num_sms", _I), ("const_sig", _I),
                ("tiles_per_unit", _I), ("kernel_kind", _I), ("acc_bits", _I), ("cond_bound", ctypes.c_double),
                ("map_floor", ctypes.c_double), ("nyquist_gain", ctypes.c_double),
                ("small_clusters", _I), ("small_cluster_ctas", _I), ("small_ctas_per_sm", _I), ("small_max", _S)]


class PLRError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        name = lib.plr_status_string(status).decode()
        detail = lib.plr_last_error().decode()
        super().__init__("%s: %s (%s)" % (where, name, detail))


def _check(status: int, where: str):
    if status != 0:
        raise PLRError(status, where)


def abi_version() -> int:
    return lib.plr_abi_version()


def _torch():
    import torch
    return torch


def _stream_ptr(stream=None):
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dev_ptr(t, dtype_name):
    torch = _torch()
    want = torch.int32 if dtype_name == "int32" else torch.float32
    if not t.is_cuda:
        raise ValueError("expected a CUDA tensor")
    if t.dtype != want:
        raise TypeError("expected %s, got %s" % (want, t.dtype))
    if not t.is_contiguous():
        raise ValueError("expected a contiguous tensor")
    return ctypes.c_void_p(t.data_ptr())


def shard_bounds(n_total: int, world: int, rank: int):
    """Contiguous rank-ordered segments (the last ranks get the remainder)."""
    base, rem = divmod(n_total, world)
    start = rank * base + max(0, rank - (world - rem))
    return start, base + (1 if rank >= world - rem else 0)


class Plan:
    """A planned recurrence (signature a : b) for one dtype and up to n_max elements."""

    def __init__(self, a, b, dtype: str = "int32", n_max: int = 1 << 30, _stages=None):
        if dtype not in _DTYPES:
            raise ValueError("dtype must be 'int32' or 'float32'")
        self.dtype = dtype
        self.n_max = int(n_max)
        self.stages = None
        h = _P()
        if _stages is None:
            self.a = tuple(float(v) for v in a)
            self.b = tuple(float(v) for v in b)
            arr_a = (ctypes.c_double * len(self.a))(*self.a)
            arr_b = (ctypes.c_double * max(1, len(self.b)))(*self.b)
            _check(lib.plr_plan_create(ctypes.byref(h), arr_a, len(self.a) - 1, arr_b, len(self.b), _DTYPES[dtype],
                                       self.n_max), "plr_plan_create")
        else:
            self.stages = tuple((tuple(float(v) for v in sa), tuple(float(v) for v in sb)) for sa, sb in _stages)
            fa = [v for sa, _ in self.stages for v in sa]
            fb = [v for _, sb in self.stages for v in sb]
            arr_a = (ctypes.c_double * max(1, len(fa)))(*fa)
            arr_b = (ctypes.c_double * max(1, len(fb)))(*fb)
            ps = (ctypes.c_int * len(self.stages))(*[len(sa) - 1 for sa, _ in self.stages])
            ks = (ctypes.c_int * len(self.stages))(*[len(sb) for _, sb in self.stages])
            _check(lib.plr_plan_create_cascade(ctypes.byref(h), len(self.stages), arr_a, ps, arr_b, ks,
                                               _DTYPES[dtype], self.n_max), "plr_plan_create_cascade")
            ca = (ctypes.c_double * 8)()
            cb = (ctypes.c_double * 8)()
            _check(lib.plr_plan_get_signature(h, ca, cb), "plr_plan_get_signature")
            pi = PlanInfo()
            _check(lib.plr_plan_get_info(h, ctypes.byref(pi)), "plr_plan_get_info")
            self.a = tuple(ca[j] for j in range(pi.p + 1))
            self.b = tuple(cb[j] for j in range(pi.k))
        self.p = len(self.a) - 1
        self.k = len(self.b)
        self._h = h
        self._hist = None
        self.device = None                      # CUDA device the plan's scratch lives on
        if self.n_max > 0:
            torch = _torch()
            if torch.cuda.is_available():
                self.device = torch.cuda.current_device()

    @classmethod
    def cascade(cls, stages, dtype: str = "int32", n_max: int = 1 << 30) -> "Plan":
        """One-pass plan of a cascade of signatures [(a_1, b_1), (a_2, b_2), ...]
        (plr_plan_create_cascade: the stages' z-transforms multiplied by the
        planner)."""
        return cls(None, None, dtype, n_max, _stages=stages)

    def signature(self):
        """(a, b) as the kernels use them (int32 residues in [0, 2^32), fp32 roundings)."""
        ca = (ctypes.c_double * 8)()
        cb = (ctypes.c_double * 8)()
        _check(lib.plr_plan_get_signature(self._h, ca, cb), "plr_plan_get_signature")
        return tuple(ca[j] for j in range(self.p + 1)), tuple(cb[j] for j in range(self.k))

    # ------------------------------------------------------------------
    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            lib.plr_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    KERNEL_NAMES = {0: "plr_scan_kernel (DECAY single-hop pipeline)", 1: "plr_scan_tmem_kernel (TMEM parking)",
                    2: "plr_scan_rr_kernel (L2 re-read)", 3: "plr_scan_kernel (generic pipeline)",
                    4: "plr_scan_dect_kernel (DECAY, map outputs parked in TMEM)"}

    def kernel_name(self) -> str:
        return self.KERNEL_NAMES.get(self.info["kernel_kind"], "?")

    @property
    def info(self) -> dict:
        pi = PlanInfo()
        _check(lib.plr_plan_get_info(self._h, ctypes.byref(pi)), "plr_plan_get_info")
        d = {f: getattr(pi, f) for f, _ in PlanInfo._fields_}
        d["cls"] = _CLASSES.get(d["cls"], str(d["cls"]))
        d["dtype"] = "int32" if d["dtype"] == 0 else "float32"
        return d

    def debug_stats(self, reset: bool = False) -> dict:
        """Look-back counters (plan created with PLR_STATS=1 in the environment)."""
        buf = (ctypes.c_uint64 * 16)()
        _check(lib.plr_plan_debug_stats(self._h, buf, int(reset)), "plr_plan_debug_stats")
        return {"lookbacks": buf[0], "windows": buf[1], "waits": buf[2], "depth_sum": buf[3],
                "cyc_agg": buf[4], "cyc_lookback": buf[5], "cyc_sleep": buf[6], "cyc_load": buf[7],
                "cyc_fold": buf[8], "trace": [buf[i] for i in range(9, 16)]}

    def factor_lists(self, m: int):
        """The k seed-extended correction-factor lists (Sec. 2.1) as planned."""
        import numpy as np
        npdt = np.int32 if self.dtype == "int32" else np.float32
        out = np.empty((self.k, self.k + m), dtype=npdt)
        _check(lib.plr_plan_factor_lists(self._h, m, out.ctypes.data_as(_P)), "plr_plan_factor_lists")
        return out

    # ------------------------------------------------------------------
    def _on_plan_device(self, *ts):
        """Every tensor must live on the device the plan was created on."""
        for t in ts:
            if t is not None and t.is_cuda and self.device is not None and t.device.index != self.device:
                raise ValueError("tensor on cuda:%d, plan created on cuda:%d" % (t.device.index, self.device))

    def _out(self, x, out):
        torch = _torch()
        if out is None:
            out = torch.empty_like(x)
        elif out.numel() != x.numel():
            raise ValueError("out has %d elements, x has %d" % (out.numel(), x.numel()))
        self._on_plan_device(x, out)
        return out

    def _hists(self, x_hist, y_hist):
        if x_hist is not None and x_hist.numel() < self.p:
            raise ValueError("x_hist needs the p = %d previous inputs" % self.p)
        if y_hist is not None and y_hist.numel() < self.k:
            raise ValueError("y_hist needs the k = %d previous outputs" % self.k)
        self._on_plan_device(x_hist, y_hist)

    @staticmethod
    def _payload_ok(payload, nbytes=PAYLOAD_BYTES):
        if payload.numel() * payload.element_size() < nbytes:
            raise ValueError("payload buffer needs %d bytes" % nbytes)
        if not payload.is_contiguous():
            raise ValueError("payload buffer must be contiguous")

    def __call__(self, x, out=None, stream=None):
        """y = recurrence(x) with zero initial conditions."""
        out = self._out(x, out)
        n = x.numel()
        _check(lib.plr_execute(self._h, _dev_ptr(x, self.dtype), _dev_ptr(out, self.dtype), n, _stream_ptr(stream)),
               "plr_execute")
        return out

    def reverse(self, x, out=None, stream=None):
        """The anticausal recurrence (Eq. (1) from the end, zero beyond it)."""
        out = self._out(x, out)
        _check(lib.plr_execute_reverse(self._h, _dev_ptr(x, self.dtype), _dev_ptr(out, self.dtype), x.numel(),
                                       _stream_ptr(stream)), "plr_execute_reverse")
        return out

    def scan_comparator(self, x, out=None, stream=None):
        """The paper's Scan comparator (Blelloch matrix-vector scan via CUB;
        a baseline, not the PLR path)."""
        out = self._out(x, out)
        _check(lib.plr_scan_comparator(self._h, _dev_ptr(x, self.dtype), _dev_ptr(out, self.dtype), x.numel(),
                                       _stream_ptr(stream)), "plr_scan_comparator")
        return out

    def bidirectional(self, x, out=None, tmp=None, stream=None):
        """Forward then backward (zero-phase) filtering; tmp holds the forward
        result (allocated when p > 0 and not given)."""
        out = self._out(x, out)
        if tmp is None and self.p > 0:
            tmp = _torch().empty_like(x)
        if tmp is not None and tmp.numel() != x.numel():
            raise ValueError("tmp must have x.numel() elements")
        self._on_plan_device(tmp)
        _check(lib.plr_execute_bidirectional(self._h, _dev_ptr(x, self.dtype), _dev_ptr(out, self.dtype), x.numel(),
                                             _dev_ptr(tmp, self.dtype) if tmp is not None else None,
                                             _stream_ptr(stream)), "plr_execute_bidirectional")
        return out

    def continue_(self, x, out=None, x_hist=None, y_hist=None, stream=None):
        """Continue a sequence from the p previous inputs and k previous outputs."""
        out = self._out(x, out)
        self._hists(x_hist, y_hist)
        xh = _dev_ptr(x_hist, self.dtype) if x_hist is not None else None
        yh = _dev_ptr(y_hist, self.dtype) if y_hist is not None else None
        _check(lib.plr_execute_continue(self._h, _dev_ptr(x, self.dtype), _dev_ptr(out, self.dtype), x.numel(),
                                        xh, yh, _stream_ptr(stream)), "plr_execute_continue")
        return out

    def reduce(self, x, payload=None, stream=None):
        """Reduce-only pass: 64-byte end-state payload of x (zero history)."""
        torch = _torch()
        if payload is None:
            payload = torch.empty(PAYLOAD_BYTES, dtype=torch.uint8, device=x.device)
        self._payload_ok(payload)
        self._on_plan_device(x, payload)
        _check(lib.plr_reduce(self._h, _dev_ptr(x, self.dtype), x.numel(), ctypes.c_void_p(payload.data_ptr()),
                              _stream_ptr(stream)), "plr_reduce")
        return payload

    def payload_from_output(self, x, y, payload=None, stream=None):
        torch = _torch()
        if payload is None:
            payload = torch.empty(PAYLOAD_BYTES, dtype=torch.uint8, device=x.device)
        if y.numel() != x.numel():
            raise ValueError("y has %d elements, x has %d" % (y.numel(), x.numel()))
        self._payload_ok(payload)
        self._on_plan_device(x, y, payload)
        _check(lib.plr_payload_from_output(self._h, _dev_ptr(x, self.dtype), _dev_ptr(y, self.dtype), x.numel(),
                                           ctypes.c_void_p(payload.data_ptr()), _stream_ptr(stream)),
               "plr_payload_from_output")
        return payload

    def combine(self, payloads, rank: int, world: int, hist=None, stream=None):
        """Boundary history of `rank` from all ranks' payloads (device)."""
        torch = _torch()
        if hist is None:                        # 8 slots x_{-4..-1}, y_{-4..-1} in the plan's dtype
            hist = torch.zeros(8, dtype=torch.int32 if self.dtype == "int32" else torch.float32,
                               device=payloads.device)
        if not 0 <= rank < world:
            raise ValueError("rank %d outside world %d" % (rank, world))
        self._payload_ok(payloads, world * PAYLOAD_BYTES)
        self._payload_ok(hist, 32)
        self._on_plan_device(payloads, hist)
        _check(lib.plr_combine(self._h, ctypes.c_void_p(payloads.data_ptr()), rank, world,
                               ctypes.c_void_p(hist.data_ptr()), _stream_ptr(stream)), "plr_combine")
        return hist

    def combine_host(self, payloads: bytes, rank: int, world: int) -> bytes:
        """Same combine on the host (no GPU): payloads = world * 64 bytes."""
        buf = ctypes.create_string_buffer(bytes(payloads), len(payloads))
        hist = ctypes.create_string_buffer(32)
        _check(lib.plr_combine_host(self._h, buf, rank, world, hist), "plr_combine_host")
        return hist.raw

    def fixup(self, y, hist, stream=None):
        self._payload_ok(hist, 32)
        self._on_plan_device(y, hist)
        _check(lib.plr_fixup(self._h, _dev_ptr(y, self.dtype), y.numel(), ctypes.c_void_p(hist.data_ptr()),
                             _stream_ptr(stream)), "plr_fixup")
        return y

    def execute_host(self, x_host, y_host=None, stream=None):
        """End to end from host memory (pinned for full speed): chunked
        H2D -> recurrence -> D2H with copies overlapped (synchronous)."""
        torch = _torch()
        if y_host is None:
            y_host = torch.empty_like(x_host, pin_memory=x_host.is_pinned())
        if x_host.is_cuda or y_host.is_cuda:
            raise ValueError("execute_host takes host tensors")
        if y_host.numel() != x_host.numel() or not x_host.is_contiguous() or not y_host.is_contiguous():
            raise ValueError("x_host / y_host must be contiguous and of equal length")
        want = _torch().int32 if self.dtype == "int32" else _torch().float32
        if x_host.dtype != want or y_host.dtype != want:
            raise TypeError("expected %s host tensors" % want)
        _check(lib.plr_execute_host(self._h, ctypes.c_void_p(x_host.data_ptr()), ctypes.c_void_p(y_host.data_ptr()),
                                    x_host.numel(), _stream_ptr(stream)), "plr_execute_host")
        return y_host

    # ------------------------------------------------------------------
    def sharded(self, x, out=None, comm: "ShardComm" = None, stream=None):
        """This rank's contiguous segment of a sequence sharded over the
        ranks of `comm` (one NCCL allgather of 64 bytes per rank)."""
        out = self._out(x, out)
        _check(lib.plr_execute_sharded(self._h, _dev_ptr(x, self.dtype), _dev_ptr(out, self.dtype), x.numel(),
                                       comm.rank, comm.world, comm.handle, _stream_ptr(stream)),
               "plr_execute_sharded")
        return out


def broadcast_bytes(payload, group=None) -> bytes:
    """Group rank 0's bytes to every rank of `group` (torch.distributed)."""
    import torch.distributed as dist
    obj = [payload if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    return obj[0]


def gather_payloads(payload: bytes, group=None) -> bytes:
    """All ranks' 64-byte payloads in rank order (host path over the process
    group; the device path uses plr_execute_sharded's NCCL allgather)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    mine = torch.frombuffer(bytearray(payload), dtype=torch.uint8)
    out = [torch.empty(PAYLOAD_BYTES, dtype=torch.uint8) for _ in range(world)]
    dist.all_gather(out, mine, group=group)
    return b"".join(bytes(t.numpy().tobytes()) for t in out)


class ShardComm:
    """NCCL communicator of the library, bootstrapped through torch.distributed:
    rank 0 creates the unique id, the process group broadcasts its bytes."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        idbuf = ctypes.create_string_buffer(128)
        if self.rank == 0:
            _check(lib.plr_nccl_unique_id(idbuf, 128), "plr_nccl_unique_id")
        idbuf = ctypes.create_string_buffer(broadcast_bytes(idbuf.raw, group), 128)
        h = _P()
        _check(lib.plr_nccl_comm_init(ctypes.byref(h), idbuf, self.rank, self.world), "plr_nccl_comm_init")
        self.handle = h

    def close(self):
        if self.handle is not None and self.handle.value:
            lib.plr_nccl_comm_destroy(self.handle)
            self.handle = None
