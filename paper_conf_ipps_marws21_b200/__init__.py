"""B200-native hot path of Adaptive Hogbatch (Ma, Rusu, Wu, Sim — IPDPSW/MARWS 2021).

Thin Python binding over the C-ABI library ``libhogbatch.so`` (``include/hogbatch.h``):
argument marshalling only — every step of the path runs in the library's CUDA kernels.
PyTorch tensors are accepted wherever device memory is needed (only ``data_ptr()``,
``stride()``, ``dtype`` and ``shape`` are read); PyTorch is plumbing, not the product.

Names follow the paper: ``mlp_create`` / ``mlp_step`` / ``mlp_loss`` / ``hogbatch_run``.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass, field

import numpy as np

from . import _lib
from ._lib import (ACTIONS, HB_ADAPTIVE, HB_BF16, HB_CREDIT_COMPLETION, HB_CREDIT_DISPATCH, HB_F32,  # noqa: F401
                   HB_HOGBATCH, HB_MINIBATCH, HB_PREC_BF16, HB_PREC_FP32_CHECK, HB_RESET_FASTEST,
                   HB_RESET_NONE, HB_STATIC, HB_UPDATE_ATOMIC, HB_UPDATE_HOGWILD, OPTIONS, HogbatchError)

lib = _lib.load()


def _check(rc: int):
    if rc != 0:
        raise HogbatchError(rc, lib.hb_last_error().decode(errors="replace"))


def device_ok(device: int = 0) -> bool:
    return bool(lib.hb_device_ok(device))


def _xdtype(t) -> int:
    s = str(t.dtype)
    if "bfloat16" in s:
        return HB_BF16
    if "float32" in s:
        return HB_F32
    raise TypeError(f"X must be bfloat16 or float32, got {s}")


def _stream_ptr(stream):
    if stream is None:
        return None
    return C.c_void_p(int(getattr(stream, "cuda_stream", stream)))


class MLP:
    """``mlp_create(dims, activation)``: the global model (fp32 master + bf16 shadow on device)."""

    def __init__(self, dims, precision: str = "bf16", seed: int = 0, device: int = 0):
        self.dims = [int(d) for d in dims]
        self.precision = precision
        self.device = device
        arr = (C.c_int32 * len(self.dims))(*self.dims)
        h = C.c_void_p()
        prec = HB_PREC_BF16 if precision == "bf16" else HB_PREC_FP32_CHECK
        _check(lib.mlp_create(arr, len(self.dims), 0, prec, seed, device, C.byref(h)))
        self.h = h

    @property
    def num_params(self) -> int:
        n = C.c_int64()
        _check(lib.mlp_num_params(self.h, C.byref(n)))
        return n.value

    def set_option(self, name: str, value: int) -> None:
        """``mlp_set_option``: a per-model setting (HB_OPT_*; names in ``OPTIONS``)."""
        _check(lib.mlp_set_option(self.h, OPTIONS[name], int(value)))

    def get_option(self, name: str) -> int:
        v = C.c_int64()
        _check(lib.mlp_get_option(self.h, OPTIONS[name], C.byref(v)))
        return v.value

    def set_fused_min_batch(self, min_batch: int) -> None:
        """Steps of >= min_batch rows take the fused row-block kernel when eligible (0 = never).
        Call before creating workers."""
        self.set_option("fused_min_batch", min_batch)

    def attach_peers(self, peers, scale: float = 1.0) -> None:
        """``mlp_attach_peers``: every update of this model also goes to each peer replica (NEXT f2)."""
        hs = (C.c_void_p * max(1, len(peers)))(*[p.h.value for p in peers])
        _check(lib.mlp_attach_peers(self.h, hs, len(peers), scale))

    def ipc_handle(self) -> bytes:
        """``mlp_ipc_handle``: 128 bytes another process passes to ``attach_ipc_peers``."""
        buf = (C.c_uint8 * 128)()
        _check(lib.mlp_ipc_handle(self.h, buf))
        return bytes(buf)

    def attach_ipc_peers(self, handles, scale: float = 1.0) -> None:
        blob = b"".join(handles)
        buf = (C.c_uint8 * max(1, len(blob)))(*blob)
        _check(lib.mlp_attach_ipc_peers(self.h, buf, len(handles), scale))

    def merge_replicas(self, workers, gamma: float = 1.0) -> None:
        """``hb_merge_replicas``: integrate the deep replicas among `workers` into this model."""
        hs = (C.c_void_p * len(workers))(*[w.h.value for w in workers])
        _check(lib.hb_merge_replicas(self.h, hs, len(workers), gamma))

    def fused_path(self, batch: int = 8192) -> int:
        """Cluster size (1, 2, 4 or 8) of the fused row-block step kernel at `batch` rows, 0 if
        steps use the per-layer GEMM chain."""
        cs = C.c_int32(0)
        r = lib.mlp_fused_path(self.h, batch, C.byref(cs))
        if r < 0:
            _check(r)
        return cs.value if r == 1 else 0

    def get_params(self, out: np.ndarray | None = None) -> np.ndarray:
        """``mlp_get_params`` into `out` (float32, num_params; pass a view of pinned host memory
        for a full-bandwidth copy) or a new array."""
        if out is None:
            out = np.empty(self.num_params, dtype=np.float32)
        if out.dtype != np.float32 or out.size != self.num_params or not out.flags["C_CONTIGUOUS"]:
            raise ValueError("out must be a contiguous float32 array of num_params elements")
        _check(lib.mlp_get_params(self.h, out.ctypes.data_as(C.POINTER(C.c_float)), out.size))
        return out

    def set_params(self, flat) -> None:
        flat = np.ascontiguousarray(flat, dtype=np.float32)
        _check(lib.mlp_set_params(self.h, flat.ctypes.data_as(C.POINTER(C.c_float)), flat.size))

    def loss(self, X, y, n: int | None = None) -> float:
        """``mlp_loss``: mean cross-entropy over the first n rows of (X, y) (device tensors)."""
        n = X.shape[0] if n is None else n
        out = C.c_double()
        _check(lib.mlp_loss(self.h, C.c_void_p(X.data_ptr()), X.stride(0), _xdtype(X),
                            C.c_void_p(y.data_ptr()), n, C.byref(out)))
        return out.value

    def merge_begin(self):
        _check(lib.hb_merge_begin(self.h))

    def merge(self, comm: "Comm", gamma: float = 1.0, stream=None):
        _check(lib.hb_merge(self.h, comm.h, gamma, _stream_ptr(stream)))

    def close(self):
        if getattr(self, "h", None):
            lib.mlp_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Worker:
    """A GPU worker (§V.A): activation scratch for max_batch rows and a stream."""

    def __init__(self, model: MLP, max_batch: int, stream=None, sub_batches: int = 1, replica: bool = False,
                 device: int | None = None):
        """sub_batches = t > 1 creates a nested worker (Alg. 2's CPU worker, L224-L235); replica=True
        a deep-replica worker (private copy of the model, merged at sync points, L134/L141)."""
        self.model = model
        self.max_batch = max_batch
        self.sub_batches = sub_batches
        self.replica = replica
        h = C.c_void_p()
        if sub_batches > 1:
            _check(lib.mlp_worker_create_nested(model.h, max_batch, sub_batches, _stream_ptr(stream), C.byref(h)))
        else:
            dev = model.device if device is None else device
            _check(lib.mlp_worker_create(model.h, dev, max_batch, int(replica), _stream_ptr(stream), C.byref(h)))
        self.h = h

    def params(self) -> np.ndarray:
        """``mlp_worker_params``: this worker's parameters (its replica's for a deep replica)."""
        out = np.empty(self.model.num_params, dtype=np.float32)
        _check(lib.mlp_worker_params(self.h, out.ctypes.data_as(C.POINTER(C.c_float)), out.size))
        return out

    @property
    def stream_handle(self) -> int:
        return lib.mlp_worker_stream(self.h) or 0

    def step(self, X, y, batch: int | None = None, lr: float = 0.1, want_loss: bool = False):
        """``mlp_step(worker, X, y, batch, lr)`` on the rows starting at X[0] / y[0]."""
        batch = X.shape[0] if batch is None else batch
        out = C.c_float()
        _check(lib.mlp_step(self.h, C.c_void_p(X.data_ptr()), X.stride(0), _xdtype(X),
                            C.c_void_p(y.data_ptr()), batch, lr, C.byref(out) if want_loss else None))
        return out.value if want_loss else None

    def step_grads(self, X, y, batch: int | None = None):
        """Test-only: gradients of the batch (flat mlp_get_params layout) and the batch loss."""
        batch = X.shape[0] if batch is None else batch
        g = np.empty(self.model.num_params, dtype=np.float32)
        out = C.c_float()
        _check(lib.mlp_step_grads(self.h, C.c_void_p(X.data_ptr()), X.stride(0), _xdtype(X),
                                  C.c_void_p(y.data_ptr()), batch,
                                  g.ctypes.data_as(C.POINTER(C.c_float)), g.size, C.byref(out)))
        return g, out.value

    def row_losses(self, n: int) -> np.ndarray:
        """Test-only: per-example cross-entropy of the first n rows of the last step."""
        out = np.empty(n, dtype=np.float32)
        _check(lib.mlp_row_losses(self.h, out.ctypes.data_as(C.POINTER(C.c_float)), n))
        return out

    def close(self):
        if getattr(self, "h", None):
            lib.mlp_worker_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


@dataclass
class WorkerSpec:
    min_b: int
    max_b: int
    init_b: int
    incr: float = 1.0
    c0: float = 0.0
    c1: float = 1.0


@dataclass
class Policy:
    """hb_policy: scheduling policy and hyperparameters held by the coordinator (L123)."""
    kind: int = HB_ADAPTIVE
    workers: list = field(default_factory=list)
    alpha: int = 2
    eta0: float = 0.1
    b0: int = 32
    reset: int = HB_RESET_FASTEST
    credit: int = HB_CREDIT_DISPATCH
    deterministic: bool = False
    eval_loss: bool = False
    max_steps: int = 0
    merges_per_epoch: int = 0
    merge_gamma: float = 1.0
    comm: "Comm | None" = None
    update: int = -1              # -1: the models' HB_OPT_UPDATE; HB_UPDATE_HOGWILD / HB_UPDATE_ATOMIC
    epoch_barrier: bool = True
    check_labels: bool = False
    coord: "Coord | None" = None  # shared cross-process coordinator
    first_worker: int = 0         # with coord: global id of this process's first worker

    def to_c(self):
        ws = (_lib.WorkerPolicy * len(self.workers))(*[
            _lib.WorkerPolicy(w.min_b, w.max_b, w.init_b, w.incr, w.c0, w.c1) for w in self.workers])
        p = _lib.Policy(self.kind, self.alpha, self.eta0, self.b0, self.reset, self.credit,
                        int(self.deterministic), int(self.eval_loss), self.max_steps,
                        self.merges_per_epoch, self.merge_gamma,
                        self.comm.h if self.comm is not None else None, len(self.workers), ws,
                        self.update, int(self.epoch_barrier), int(self.check_labels),
                        self.coord.h if self.coord is not None else None, self.first_worker)
        return p, ws


@dataclass
class CSR:
    """A sparse data set for hogbatch_run (hb_dataset format HB_DATA_CSR): torch tensors, all on the
    host (pinned for an asynchronous copy) or all on the device; densified on the device into rows
    of `ldx` (default: n_cols rounded up to 8) elements ("processed in dense format")."""
    indptr: object   # int64 [n + 1]
    indices: object  # int32 [nnz]
    values: object   # bfloat16 (bf16 models) or float32 [nnz]
    n_cols: int
    ldx: int = 0

    @property
    def n(self) -> int:
        return self.indptr.numel() - 1


def _dataset(X, y, n):
    if isinstance(X, CSR):
        ld = X.ldx or pad_to(X.n_cols)
        n = X.n if n is None else n
        return _lib.Dataset(None, ld, _xdtype(X.values), y.data_ptr(), n, _lib.HB_DATA_CSR, X.n_cols,
                            X.indptr.data_ptr(), X.indices.data_ptr(), X.values.data_ptr()), n
    n = X.shape[0] if n is None else n
    return _lib.Dataset(X.data_ptr(), X.stride(0), _xdtype(X), y.data_ptr(), n, _lib.HB_DATA_DENSE, 0, None, None,
                        None), n


def _rec_tuple(r):
    return (r.seq, r.epoch, r.worker, r.vtime, r.u_before, r.b_before, ACTIONS[r.action], r.b_after,
            r.u_after, r.served, r.offset, r.lr)


def schedule_trace(policy: Policy, N: int, epochs: int, cap: int = 1 << 20):
    """``hb_schedule_trace``: the coordinator on the virtual clock (no GPU needed)."""
    p, _keep = policy.to_c()
    buf = (_lib.TraceRec * cap)()
    n = C.c_int64()
    _check(lib.hb_schedule_trace(C.byref(p), N, epochs, buf, cap, C.byref(n)))
    return [_rec_tuple(buf[i]) for i in range(min(n.value, cap))]


def hogbatch_run(workers, policy: Policy, X, y, epochs: int = 1, n: int | None = None,
                 trace_cap: int = 0, step_loss_cap: int = 0, max_epochs: int | None = None,
                 train_loss: bool = False):
    """``hogbatch_run(workers, policy, epochs)`` over X [N x ldx] (device, or pinned host memory staged by
    the library) or a ``CSR`` data set, labels y [N].  Per-worker statistics are indexed by the global
    worker id (policy.workers)."""
    ds, n = _dataset(X, y, n)
    p, _keep = policy.to_c()
    W = len(policy.workers)
    me = max_epochs or epochs
    el = (C.c_double * me)()
    et = (C.c_double * me)()
    up = (C.c_int64 * (me * W))()
    sm = (C.c_int64 * (me * W))()
    tr = (_lib.TraceRec * max(trace_cap, 1))()
    sl = (C.c_float * max(step_loss_cap, 1))()
    st = _lib.Stats(me, 0, el, et, up, sm, tr, trace_cap, 0, sl, step_loss_cap, 0, 0.0, 0, 0, int(train_loss), 0.0)
    hs = (C.c_void_p * len(workers))(*[w.h.value for w in workers])
    _check(lib.hogbatch_run(hs, len(workers), C.byref(p), C.byref(ds), epochs, C.byref(st)))
    ed = st.epochs_done
    return dict(
        epochs_done=ed,
        epoch_loss=[el[i] for i in range(min(ed, me))],
        epoch_train_s=[et[i] for i in range(min(ed, me))],
        updates=np.array([up[i] for i in range(me * W)]).reshape(me, W)[:max(ed, 1)],
        samples=np.array([sm[i] for i in range(me * W)]).reshape(me, W)[:max(ed, 1)],
        trace=[_rec_tuple(tr[i]) for i in range(min(st.trace_len, trace_cap))],
        trace_len=st.trace_len,
        step_loss=[sl[i] for i in range(min(st.n_steps, step_loss_cap))],
        n_steps=st.n_steps,
        total_train_s=st.total_train_s,
        total_samples=st.total_samples,
        n_merges=st.n_merges,
        train_loss=st.train_loss,
    )


class Coord:
    """``hb_coord_create``: the node's shared coordinator (POSIX shared memory `name`); rank 0
    creates it, the other ranks attach.  Pass as Policy.coord with Policy.first_worker."""

    def __init__(self, name: str, policy: Policy, N: int, nranks: int, rank: int):
        p, _keep = policy.to_c()
        h = C.c_void_p()
        _check(lib.hb_coord_create(name.encode(), C.byref(p), N, nranks, rank, C.byref(h)))
        self.h = h

    def reset(self, policy: Policy, N: int):
        p, _keep = policy.to_c()
        _check(lib.hb_coord_reset(self.h, C.byref(p), N))

    def schedule(self, worker: int, now: float):
        """One ScheduleWork(worker) on the shared state (test / custom-driver entry)."""
        r = _lib.TraceRec()
        _check(lib.hb_coord_schedule(self.h, worker, now, C.byref(r)))
        return _rec_tuple(r)

    def idle(self, worker: int) -> bool:
        """The worker could not be served; True if every worker now idles (the epoch ended)."""
        e = C.c_int32()
        _check(lib.hb_coord_idle(self.h, worker, C.byref(e)))
        return bool(e.value)

    def close(self):
        if getattr(self, "h", None):
            lib.hb_coord_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Comm:
    """NCCL communicator for the replica merge (one rank per GPU)."""

    @staticmethod
    def unique_id() -> bytes:
        buf = (C.c_uint8 * 128)()
        _check(lib.hb_nccl_unique_id(buf))
        return bytes(buf)

    def __init__(self, uid: bytes, nranks: int, rank: int, device: int):
        buf = (C.c_uint8 * 128)(*uid)
        h = C.c_void_p()
        _check(lib.hb_comm_create(buf, nranks, rank, device, C.byref(h)))
        self.h = h

    def close(self):
        if getattr(self, "h", None):
            lib.hb_comm_destroy(self.h)
            self.h = None


def kernel_launches() -> int:
    """Kernels this library has launched in this process."""
    return int(lib.hb_kernel_launches())


def prof_enable(on: bool = True):
    _check(lib.hb_prof_enable(int(on)))


def prof_read(reset: bool = False, per_layer: bool = False) -> dict:
    """Per kernel class: launches, device ms, algorithmic flops and bytes (blocking).
    per_layer=True also returns "<class>/l<k>" entries (weight layer k, 0-based) with launches."""
    nc, nl = len(_lib.PROF_CLASSES), _lib.PROF_LAYERS
    buf = (_lib.ProfEntry * (nc * (1 + nl)))()
    _check(lib.hb_prof_read(buf, nc * (1 + nl), int(reset)))

    def ent(e):
        return dict(launches=e.launches, ms=e.ms, flops=e.flops, bytes=e.bytes)
    out = {name: ent(buf[i]) for i, name in enumerate(_lib.PROF_CLASSES)}
    if per_layer:
        for c, name in enumerate(_lib.PROF_CLASSES):
            for k in range(nl):
                e = buf[nc + c * nl + k]
                if e.launches:
                    out[f"{name}/l{k}"] = ent(e)
    return out


def pad_to(n: int, m: int = 8) -> int:
    return (n + m - 1) // m * m
