"""Thin ctypes binding of the C-ABI in include/occu.h (argument marshalling only).

Every step of the hot path runs in ``lib/libocc_b200.so``; this module never
computes anything itself and raises if the library is missing.  Arrays may be
NumPy (host memory; calls are synchronous) or CUDA torch tensors (device
memory; calls are stream-ordered on the ctx stream, by default torch's current
stream).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "lib", "libocc_b200.so")

OCCU_OK, OCCU_EINVAL, OCCU_ENOMEM, OCCU_ECUDA, OCCU_EFORMAT, OCCU_ENOTREADY, OCCU_ENCCL = range(7)
AGGR_SUM, AGGR_MEAN = 0, 1
MSG_CHANNEL_SOFTMAX, MSG_NEIGHBOR_SOFTMAX = 0, 1
FP32, BF16 = 0, 1
T_HBAR, T_P, T_Q, T_E, T_H, T_R, T_YHAT, T_GPH = range(8)
STATUS_NAMES = {0: "OK", 1: "EINVAL", 2: "ENOMEM", 3: "ECUDA", 4: "EFORMAT", 5: "ENOTREADY",
                6: "ENCCL"}

EXPORTS = [
    "occu_create", "occu_destroy", "occu_set_stream", "occu_num_params", "occu_init_weights",
    "occu_load_weights", "occu_save_weights", "occu_set_params", "occu_get_params", "occu_pack",
    "occu_batch_to_device", "occu_batch_free", "occu_predict", "occu_train_step",
    "occu_compute_grads", "occu_get_grads", "occu_set_weight_decay", "occu_nccl_unique_id",
    "occu_dist_init", "occu_save_state", "occu_load_state", "occu_set_keep_intermediates",
    "occu_get_tensor", "occu_last_launch_count", "occu_last_error", "occu_set_profiling",
    "occu_profile_reset", "occu_profile_query", "occu_set_kernel_path", "occu_pack_jobs",
    "occu_template_create", "occu_template_destroy", "occu_synthesize", "occu_set_small_batch_kernel",
    "occu_dist_set_timeout", "occu_dist_abort", "occu_dist_sync", "occu_train_step_async",
]


class OccuError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"occu status {STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class Config(C.Structure):
    _fields_ = [("L", C.c_int32), ("F_n", C.c_int32), ("F_e", C.c_int32), ("d", C.c_int32),
                ("d_h", C.c_int32), ("aggr", C.c_int32), ("msg", C.c_int32), ("prec", C.c_int32),
                ("slope", C.c_float), ("readout", C.c_int32), ("k", C.c_int32),
                ("heads", C.c_int32), ("graphormer", C.c_int32)]


class GraphView(C.Structure):
    _fields_ = [("num_nodes", C.c_int32), ("num_edges", C.c_int32),
                ("src", C.POINTER(C.c_int32)), ("dst", C.POINTER(C.c_int32))]


class CsrBatch(C.Structure):
    _fields_ = [("num_graphs", C.c_int32), ("num_nodes", C.c_int32), ("num_edges", C.c_int32),
                ("node_off", C.POINTER(C.c_int32)), ("edge_off", C.POINTER(C.c_int32)),
                ("in_ptr", C.POINTER(C.c_int32)), ("in_src", C.POINTER(C.c_int32)),
                ("in_dst", C.POINTER(C.c_int32)), ("in_eid", C.POINTER(C.c_int32)),
                ("out_ptr", C.POINTER(C.c_int32)), ("out_pos", C.POINTER(C.c_int32)),
                ("node_graph", C.POINTER(C.c_int32)), ("on_device", C.c_int32),
                ("max_in_degree", C.c_int32), ("priv", C.c_void_p)]


class BatchStruct(C.Structure):
    _fields_ = [("csr", C.POINTER(CsrBatch)), ("node_feat", C.c_void_p),
                ("edge_feat", C.c_void_p), ("global_num_graphs", C.c_int32)]


_lib = None


def lib():
    """Load the library; raise (never fall back) if it is missing."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = C.CDLL(LIB_PATH)
        P, VP, I32, U64, SZ = C.POINTER, C.c_void_p, C.c_int32, C.c_uint64, C.c_size_t
        sig = {
            "occu_create": ([P(VP), P(Config), C.c_int, VP], I32),
            "occu_destroy": ([VP], I32),
            "occu_set_stream": ([VP, VP], I32),
            "occu_num_params": ([P(Config)], SZ),
            "occu_init_weights": ([VP, U64], I32),
            "occu_load_weights": ([VP, C.c_char_p], I32),
            "occu_save_weights": ([VP, C.c_char_p], I32),
            "occu_set_params": ([VP, VP, SZ], I32),
            "occu_get_params": ([VP, VP, SZ], I32),
            "occu_pack": ([P(GraphView), I32, P(P(CsrBatch))], I32),
            "occu_pack_jobs": ([P(C.c_float), I32, C.c_double, P(I32), P(C.c_double), P(I32)], I32),
            "occu_template_create": ([VP, P(GraphView), VP, VP, VP, VP, P(VP)], I32),
            "occu_template_destroy": ([VP], None),
            "occu_synthesize": ([VP, P(VP), I32, VP, P(P(CsrBatch)), P(VP), P(VP)], I32),
            "occu_batch_to_device": ([VP, P(CsrBatch), P(P(CsrBatch))], I32),
            "occu_batch_free": ([P(CsrBatch)], None),
            "occu_predict": ([VP, P(CsrBatch), VP, VP, VP], I32),
            "occu_predict_async": ([VP, P(CsrBatch), VP, VP, VP], I32),
            "occu_wait": ([VP], I32),
            "occu_train_step": ([VP, P(BatchStruct), VP, C.c_float, P(C.c_float)], I32),
            "occu_train_step_async": ([VP, P(BatchStruct), VP, C.c_float, VP], I32),
            "occu_compute_grads": ([VP, P(BatchStruct), VP, P(C.c_float)], I32),
            "occu_get_grads": ([VP, VP, SZ], I32),
            "occu_set_weight_decay": ([VP, C.c_float], I32),
            "occu_nccl_unique_id": ([VP], I32),
            "occu_dist_init": ([VP, C.c_int, C.c_int, VP], I32),
            "occu_dist_set_timeout": ([VP, C.c_double], I32),
            "occu_dist_abort": ([VP], I32),
            "occu_dist_sync": ([VP], I32),
            "occu_save_state": ([VP, C.c_char_p], I32),
            "occu_load_state": ([VP, C.c_char_p], I32),
            "occu_set_keep_intermediates": ([VP, C.c_int], I32),
            "occu_get_tensor": ([VP, I32, I32, VP, SZ], I32),
            "occu_last_launch_count": ([VP], C.c_int64),
            "occu_test_wgrad": ([VP, VP, I32, VP, I32, C.c_int64, I32, VP], I32),
            "occu_last_error": ([VP], C.c_char_p),
            "occu_set_profiling": ([VP, C.c_int], I32),
            "occu_set_kernel_path": ([VP, C.c_int], I32),
            "occu_set_small_batch_kernel": ([VP, C.c_int], I32),
            "occu_profile_reset": ([VP], I32),
            "occu_profile_query": ([VP, I32, P(C.c_char_p), P(C.c_double), P(C.c_int64)], I32),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _check(status, ctx=None):
    if status != OCCU_OK:
        msg = lib().occu_last_error(ctx)
        raise OccuError(status, msg.decode() if msg else "")


def _ptr(x):
    """(pointer, is_device, keepalive) for a NumPy array or torch tensor."""
    if x is None:
        return None, False, None
    if isinstance(x, np.ndarray):
        x = np.ascontiguousarray(x, dtype=np.float32)
        return x.ctypes.data, False, x
    # torch tensor
    if not x.is_contiguous():
        raise ValueError("tensor must be contiguous")
    return x.data_ptr(), bool(x.is_cuda), x


READOUT_MEAN, READOUT_SET_DECODER = 0, 1


def config(L=3, F_n=80, F_e=4, d=128, d_h=None, aggr=AGGR_SUM, msg=MSG_CHANNEL_SOFTMAX,
           prec=FP32, slope=0.01, readout=READOUT_MEAN, k=4, heads=4, graphormer=0):
    return Config(L, F_n, F_e, d, d if d_h is None else d_h, aggr, msg, prec, slope, readout,
                  k if readout else 0, heads if (readout or graphormer) else 0, graphormer)


def num_params(cfg: Config) -> int:
    return int(lib().occu_num_params(C.byref(cfg)))


class Template:
    """A device-resident family template (occu_template, NEXT-4); freed on deletion."""

    def __init__(self, model, t):
        node_static = np.ascontiguousarray(t.node_static, dtype=np.float32)
        node_coef = np.ascontiguousarray(t.node_coef, dtype=np.float64)
        edge_static = np.ascontiguousarray(t.edge_static, dtype=np.float32)
        edge_coef = np.ascontiguousarray(t.edge_coef, dtype=np.float64)
        src = np.ascontiguousarray(t.src, dtype=np.int32)
        dst = np.ascontiguousarray(t.dst, dtype=np.int32)
        view = GraphView(int(t.num_nodes), len(src), src.ctypes.data_as(C.POINTER(C.c_int32)),
                         dst.ctypes.data_as(C.POINTER(C.c_int32)))
        self._p = C.c_void_p()
        self.family = t.family
        self.num_nodes, self.num_edges = int(t.num_nodes), len(src)
        _check(lib().occu_template_create(model._ctx, C.byref(view), node_static.ctypes.data,
                                          node_coef.ctypes.data, edge_static.ctypes.data,
                                          edge_coef.ctypes.data, C.byref(self._p)), model._ctx)

    def __del__(self):
        if getattr(self, "_p", None) and self._p.value and _lib is not None:
            _lib.occu_template_destroy(self._p)
            self._p = C.c_void_p()


class Csr:
    """A packed batch (occu_csr_batch), host or device; freed on deletion."""

    def __init__(self, ptr):
        self._p = ptr

    @property
    def struct(self):
        return self._p.contents

    @property
    def num_graphs(self):
        return self.struct.num_graphs

    @property
    def num_nodes(self):
        return self.struct.num_nodes

    @property
    def num_edges(self):
        return self.struct.num_edges

    @property
    def on_device(self):
        return bool(self.struct.on_device)

    def node_off_tensor(self, device: int = 0):
        """Zero-copy int32 CUDA tensor view of node_off [B + 1] (device batches only)."""
        import torch
        s = self.struct
        if not s.on_device:
            raise ValueError("host batch")
        ptr = C.cast(s.node_off, C.c_void_p).value
        return torch.as_tensor(_DeviceArray(ptr, (s.num_graphs + 1,), "<i4"),
                               device=torch.device("cuda", device))

    def arrays(self):
        """Host arrays as NumPy copies (host batches only)."""
        s = self.struct
        if s.on_device:
            raise ValueError("device batch")
        B, N, E = s.num_graphs, s.num_nodes, s.num_edges
        take = lambda p, n: np.ctypeslib.as_array(p, shape=(n,)).copy() if n else np.zeros(0, np.int32)
        return {"node_off": take(s.node_off, B + 1), "edge_off": take(s.edge_off, B + 1),
                "in_ptr": take(s.in_ptr, N + 1), "in_src": take(s.in_src, E),
                "in_dst": take(s.in_dst, E), "in_eid": take(s.in_eid, E),
                "out_ptr": take(s.out_ptr, N + 1), "out_pos": take(s.out_pos, E),
                "node_graph": take(s.node_graph, N), "num_graphs": B, "num_nodes": N,
                "num_edges": E}

    def __del__(self):
        if getattr(self, "_p", None) is not None and _lib is not None:
            _lib.occu_batch_free(self._p)
            self._p = None


_VIEW_DT = np.dtype([("num_nodes", "<i4"), ("num_edges", "<i4"), ("src", "<u8"), ("dst", "<u8")],
                    align=True)


def pack(graphs) -> Csr:
    """graphs: list of (num_nodes, src int32[m], dst int32[m]) with local ids.

    Builds the occu_graph_view array with NumPy (one concatenation, pointer
    arithmetic) and calls occu_pack; packing itself runs in the library."""
    n = len(graphs)
    assert ctypes_view_ok()
    nn = np.fromiter((g[0] for g in graphs), dtype=np.int32, count=n)
    m = np.fromiter((len(g[1]) for g in graphs), dtype=np.int64, count=n)
    src = np.concatenate([np.asarray(g[1], dtype=np.int32) for g in graphs]) if n else np.zeros(0, np.int32)
    dst = np.concatenate([np.asarray(g[2], dtype=np.int32) for g in graphs]) if n else np.zeros(0, np.int32)
    src = np.ascontiguousarray(src)
    dst = np.ascontiguousarray(dst)
    off = np.concatenate([[0], np.cumsum(m)[:-1]]).astype(np.uint64) * np.uint64(4)
    views = np.zeros(max(n, 1), dtype=_VIEW_DT)
    views["num_nodes"][:n] = nn
    views["num_edges"][:n] = m.astype(np.int32)
    views["src"][:n] = np.uint64(src.ctypes.data) + off
    views["dst"][:n] = np.uint64(dst.ctypes.data) + off
    out = C.POINTER(CsrBatch)()
    _check(lib().occu_pack(views.ctypes.data_as(C.POINTER(GraphView)), n, C.byref(out)))
    return Csr(out)


def pack_arrays(num_nodes, num_edges, src, dst) -> Csr:
    """occu_pack for a batch already held as concatenated arrays (a data loader's layout):
    num_nodes, num_edges int [B]; src, dst int32 [E] local ids, graphs back to back.  The
    occu_graph_view array is pointer arithmetic over the two arrays (no per-graph Python)."""
    nn = np.ascontiguousarray(num_nodes, dtype=np.int32)
    m = np.ascontiguousarray(num_edges, dtype=np.int64)
    n = len(nn)
    src = np.ascontiguousarray(src, dtype=np.int32)
    dst = np.ascontiguousarray(dst, dtype=np.int32)
    if len(m) != n or int(m.sum()) != len(src) or len(src) != len(dst):
        raise ValueError("num_edges must sum to len(src) == len(dst)")
    off = np.zeros(max(n, 1), np.uint64)
    if n > 1:
        off[1:n] = np.cumsum(m[:-1]).astype(np.uint64) * np.uint64(4)
    views = np.zeros(max(n, 1), dtype=_VIEW_DT)
    views["num_nodes"][:n] = nn
    views["num_edges"][:n] = m.astype(np.int32)
    views["src"][:n] = np.uint64(src.ctypes.data) + off[:n]
    views["dst"][:n] = np.uint64(dst.ctypes.data) + off[:n]
    out = C.POINTER(CsrBatch)()
    _check(lib().occu_pack(views.ctypes.data_as(C.POINTER(GraphView)), n, C.byref(out)))
    return Csr(out)


def pack_jobs(occ, capacity=1.0):
    """occu-packing (NEXT-4, P390-P392): first-fit slots for jobs by predicted occupancy.
    Returns (slot_of_job int32 [n], slot_load float64 [num_slots])."""
    occ = np.ascontiguousarray(occ, dtype=np.float32)
    n = len(occ)
    slot = np.empty(max(n, 1), np.int32)
    load = np.empty(max(n, 1), np.float64)
    ns = C.c_int32(0)
    _check(lib().occu_pack_jobs(occ.ctypes.data_as(C.POINTER(C.c_float)), n, float(capacity),
                                slot.ctypes.data_as(C.POINTER(C.c_int32)),
                                load.ctypes.data_as(C.POINTER(C.c_double)), C.byref(ns)))
    return slot[:n], load[:ns.value].copy()


class _DeviceArray:
    """Zero-copy view of library-owned device memory (__cuda_array_interface__, float32)."""

    def __init__(self, ptr, shape, typestr="<f4"):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr,
                                         "data": (int(ptr or 0), False), "version": 3}


def ctypes_view_ok() -> bool:
    return _VIEW_DT.itemsize == C.sizeof(GraphView)


class Model:
    """One occu_ctx: weights, Adam state, workspace, NCCL communicator."""

    def __init__(self, cfg: Config, device: int = 0, stream=None):
        self.cfg = cfg
        self._device = device
        self._inflight = []
        self._ctx = C.c_void_p()
        if stream is None:
            try:
                import torch
                if torch.cuda.is_available():
                    stream = torch.cuda.current_stream(device).cuda_stream
            except Exception:
                stream = None
        _check(lib().occu_create(C.byref(self._ctx), C.byref(cfg), device, stream))
        self.n_params = num_params(cfg)

    @property
    def ctx(self):
        return self._ctx

    def close(self):
        if self._ctx:
            lib().occu_destroy(self._ctx)
            self._ctx = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_stream(self, stream_handle):
        _check(lib().occu_set_stream(self._ctx, stream_handle), self._ctx)

    # weights
    def init_weights(self, seed: int):
        _check(lib().occu_init_weights(self._ctx, seed), self._ctx)

    def load_weights(self, path: str):
        _check(lib().occu_load_weights(self._ctx, path.encode()), self._ctx)

    def save_weights(self, path: str):
        _check(lib().occu_save_weights(self._ctx, path.encode()), self._ctx)

    def set_params(self, flat: np.ndarray):
        flat = np.ascontiguousarray(flat, dtype=np.float32)
        _check(lib().occu_set_params(self._ctx, flat.ctypes.data, flat.size), self._ctx)

    def get_params(self) -> np.ndarray:
        out = np.empty(self.n_params, np.float32)
        _check(lib().occu_get_params(self._ctx, out.ctypes.data, out.size), self._ctx)
        return out

    def get_grads(self) -> np.ndarray:
        out = np.empty(self.n_params, np.float32)
        _check(lib().occu_get_grads(self._ctx, out.ctypes.data, out.size), self._ctx)
        return out

    def set_weight_decay(self, wd: float):
        _check(lib().occu_set_weight_decay(self._ctx, wd), self._ctx)

    def save_state(self, path):
        _check(lib().occu_save_state(self._ctx, path.encode()), self._ctx)

    def load_state(self, path):
        _check(lib().occu_load_state(self._ctx, path.encode()), self._ctx)

    # batches
    def set_small_batch_kernel(self, enable: bool):
        _check(lib().occu_set_small_batch_kernel(self._ctx, int(bool(enable))), self._ctx)

    # NEXT-4: on-device feature synthesis
    def template(self, t):
        """Upload one family template (occu_gen.templates.Template) to this ctx's device."""
        return Template(self, t)

    def synthesize(self, templates, hp):
        """occu_synthesize: the batch of graphs templates[b] at hp[b] = (batch, cin, seq, hw),
        built on the device.  Returns (device Csr, node_feat, edge_feat) with the features as
        zero-copy CUDA tensors over library memory, valid until the next synthesize call."""
        import torch
        hp = np.ascontiguousarray(hp, dtype=np.float32).reshape(-1, 4)
        arr = (C.c_void_p * len(templates))(*[tp._p for tp in templates])
        out = C.POINTER(CsrBatch)()
        nf, ef = C.c_void_p(), C.c_void_p()
        _check(lib().occu_synthesize(self._ctx, arr, len(templates), hp.ctypes.data, C.byref(out),
                                     C.byref(nf), C.byref(ef)), self._ctx)
        csr = Csr(out)
        N, E = csr.struct.num_nodes, csr.struct.num_edges
        dev = torch.device("cuda", self._device)
        nft = torch.as_tensor(_DeviceArray(nf.value, (N, 80)), device=dev)
        eft = torch.as_tensor(_DeviceArray(ef.value, (E, 4)), device=dev)
        return csr, nft, eft

    def to_device(self, csr: Csr) -> Csr:
        out = C.POINTER(CsrBatch)()
        _check(lib().occu_batch_to_device(self._ctx, csr._p, C.byref(out)), self._ctx)
        return Csr(out)

    def predict(self, csr: Csr, node_feat, edge_feat, out=None):
        nf, dev, k1 = _ptr(node_feat)
        ef, _, k2 = _ptr(edge_feat)
        if out is None:
            if dev:
                import torch
                out = torch.empty(csr.num_graphs, dtype=torch.float32, device=node_feat.device)
            else:
                out = np.empty(csr.num_graphs, np.float32)
        op, _, k3 = _ptr(out)
        _check(lib().occu_predict(self._ctx, csr._p, nf, ef, op), self._ctx)
        return out

    def predict_async(self, csr: Csr, node_feat, edge_feat, out):
        """occu_predict_async: host batch, pinned host features and output; returns at once.
        The arguments are kept referenced until wait() (the library reads them later)."""
        nf, dev, k1 = _ptr(node_feat)
        ef, _, k2 = _ptr(edge_feat)
        op, _, k3 = _ptr(out)
        _check(lib().occu_predict_async(self._ctx, csr._p, nf, ef, op), self._ctx)
        # the previous calls' inputs are free once this call returns (the library waits for
        # their H2D copies); every output stays referenced until wait() (its D2H may be in
        # flight).  Strip the earlier entries to their outputs, then append this call in full.
        self._inflight = ([(None, None, None, None, None, None, x[6]) for x in self._inflight]
                          + [(csr, k1, k2, k3, node_feat, edge_feat, out)])
        return out

    def wait(self):
        _check(lib().occu_wait(self._ctx), self._ctx)
        self._inflight.clear()

    def _batch(self, csr, node_feat, edge_feat, global_num_graphs):
        nf, _, k1 = _ptr(node_feat)
        ef, _, k2 = _ptr(edge_feat)
        b = BatchStruct(csr._p, nf, ef, int(global_num_graphs or csr.num_graphs))
        return b, (k1, k2)

    def train_step(self, csr: Csr, node_feat, edge_feat, targets, lr: float,
                   global_num_graphs=None, want_loss=True):
        b, keep = self._batch(csr, node_feat, edge_feat, global_num_graphs)
        tp, _, k3 = _ptr(targets)
        loss = C.c_float(0.0)
        _check(lib().occu_train_step(self._ctx, C.byref(b), tp, lr,
                                     C.byref(loss) if want_loss else None), self._ctx)
        return float(loss.value) if want_loss else None

    def train_step_async(self, csr: Csr, node_feat, edge_feat, targets, lr: float,
                         global_num_graphs=None, out_loss=None):
        """occu_train_step_async: host batch, pinned host features / targets; returns at once.
        out_loss: optional pinned 1-element float32 tensor, valid after wait().  The arguments
        stay referenced until the next call (inputs) or wait() (out_loss)."""
        b, keep = self._batch(csr, node_feat, edge_feat, global_num_graphs)
        tp, _, k3 = _ptr(targets)
        lp = out_loss.data_ptr() if out_loss is not None else None
        _check(lib().occu_train_step_async(self._ctx, C.byref(b), tp, lr, lp), self._ctx)
        self._inflight = ([(None, None, None, None, None, None, x[6]) for x in self._inflight]
                          + [(csr, keep, k3, b, node_feat, edge_feat, out_loss)])

    def compute_grads(self, csr: Csr, node_feat, edge_feat, targets, global_num_graphs=None):
        b, keep = self._batch(csr, node_feat, edge_feat, global_num_graphs)
        tp, _, k3 = _ptr(targets)
        loss = C.c_float(0.0)
        _check(lib().occu_compute_grads(self._ctx, C.byref(b), tp, C.byref(loss)), self._ctx)
        return float(loss.value)

    # distributed
    @staticmethod
    def nccl_unique_id() -> bytes:
        buf = (C.c_ubyte * 128)()
        _check(lib().occu_nccl_unique_id(buf))
        return bytes(buf)

    def dist_init(self, rank: int, world: int, uid: bytes):
        buf = (C.c_ubyte * 128).from_buffer_copy(uid)
        _check(lib().occu_dist_init(self._ctx, rank, world, buf), self._ctx)

    def dist_set_timeout(self, seconds: float):
        _check(lib().occu_dist_set_timeout(self._ctx, float(seconds)), self._ctx)

    def dist_abort(self):
        _check(lib().occu_dist_abort(self._ctx), self._ctx)

    def dist_sync(self):
        _check(lib().occu_dist_sync(self._ctx), self._ctx)

    def set_kernel_path(self, path: int):
        """0 = tensor cores (default), 1 = CUDA-core SIMT FP32, 2 = tensor cores with the
        gate + aggregation fused."""
        _check(lib().occu_set_kernel_path(self._ctx, int(path)), self._ctx)

    # introspection
    def keep_intermediates(self, keep=True):
        _check(lib().occu_set_keep_intermediates(self._ctx, int(keep)), self._ctx)

    def get_tensor(self, which: int, layer: int, shape) -> np.ndarray:
        out = np.empty(shape, np.float32)
        _check(lib().occu_get_tensor(self._ctx, which, layer, out.ctypes.data, out.nbytes), self._ctx)
        return out

    def test_wgrad(self, X, Y, out, y_bf16=False):
        """Test hook: out[A][Bn] = Xᵀ Y through the backward's weight-gradient kernels
        (torch CUDA tensors: X fp32 [R][A], Y fp32 or bf16 [R][Bn], out fp32 [A][Bn])."""
        R, A = X.shape
        Bn = Y.shape[1]
        for t in (X, Y, out):
            if not (t.is_cuda and t.is_contiguous()):
                raise ValueError("contiguous CUDA tensors expected")
        _check(lib().occu_test_wgrad(self._ctx, X.data_ptr(), A, Y.data_ptr(), Bn, R,
                                     int(y_bf16), out.data_ptr()), self._ctx)
        return out

    def last_launch_count(self) -> int:
        return int(lib().occu_last_launch_count(self._ctx))

    # per-kernel CUDA-event timing
    def set_profiling(self, on=True):
        _check(lib().occu_set_profiling(self._ctx, int(on)), self._ctx)

    def profile_reset(self):
        _check(lib().occu_profile_reset(self._ctx), self._ctx)

    def profile(self) -> dict:
        """{kernel name: (total_ms, launches)} since the last reset."""
        out = {}
        i = 0
        while True:
            name = C.c_char_p()
            ms = C.c_double()
            cnt = C.c_int64()
            st = lib().occu_profile_query(self._ctx, i, C.byref(name), C.byref(ms), C.byref(cnt))
            if st != OCCU_OK:
                break
            out[name.value.decode()] = (ms.value, cnt.value)
            i += 1
        return out
