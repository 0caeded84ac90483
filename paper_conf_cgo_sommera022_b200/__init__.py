"""B200-native batched Sum-Product Network inference (the data-parallel hot
path of SPNC, Sommer et al., CGO'22).

Thin ctypes binding over ``libspnb.so`` (C ABI in ``include/spnb.h``): argument
marshalling only -- every step of inference runs in the library's sm_100a
kernels.  PyTorch is used for device memory and streams.  There is no CPU
fallback: if the library is missing, importing the binding's entry points
raises.

    g = Graph(flat_spn)                 # validate + copy   (spn_load_graph)
    plan = Plan(g)                      # prepare + upload  (spn_prepare)
    logp, am = plan.infer(x_cuda)       # joint             (spn_infer_joint)
    logp, am = plan.infer(x_cuda, marginal=True)   # NaN = missing
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from .build import LIB as _LIB_PATH

__all__ = ["SPNError", "Graph", "Plan", "load_library", "partition_graph",
           "build_program", "build_layered", "build_layered2", "LSTEP_DTYPE", "R2STEP_DTYPE", "NODE_DTYPE", "REC_DTYPE", "EDGE_DTYPE",
           "GAUSSIAN", "CATEGORICAL", "HISTOGRAM", "SUM", "PRODUCT"]

GAUSSIAN, CATEGORICAL, HISTOGRAM, SUM, PRODUCT = 0, 1, 2, 3, 4

NODE_DTYPE = np.dtype([("kind", "<i4"), ("feature", "<i4"), ("child_begin", "<i8"),
                       ("param_begin", "<i8"), ("n_children", "<i4"), ("n_params", "<i4")])
assert NODE_DTYPE.itemsize == 32
REC_DTYPE = np.dtype([("x", "<u4"), ("y", "<u4"), ("z", "<u4"), ("w", "<u4")])
EDGE_DTYPE = np.dtype([("a", "<u4"), ("b", "<u4"), ("lw", "<f4"), ("pad", "<u4")])
LSTEP_DTYPE = np.dtype([(n, "<i4") for n in ("type", "n_out", "na", "nb", "buf_a", "buf_b",
                                             "buf_out", "k_pad", "s_per_group", "n_groups",
                                             "n_group", "n_vars")] +
                       [(n, "<i8") for n in ("vars_off", "par_off", "cst_off", "w_off",
                                             "w_group_bytes")] +
                       [("rep", "<i4"), ("pad_", "<i4")])

_STATUS = {0: "SPN_OK", -1: "SPN_E_ARG", -2: "SPN_E_GRAPH", -3: "SPN_E_CUDA",
           -4: "SPN_E_OOM", -5: "SPN_E_UNSUPPORTED"}


class SPNError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_STATUS.get(code, code)}: {msg}")
        self.code = code


class _Options(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("block_threads", ctypes.c_int32),
                ("samples_per_thread", ctypes.c_int32), ("layered_path", ctypes.c_int32),
                ("max_task_nodes", ctypes.c_int64), ("tc_precision", ctypes.c_int32),
                ("ctas_per_sm", ctypes.c_int32), ("compiled_path", ctypes.c_int32),
                ("layered_kernel", ctypes.c_int32), ("value_space", ctypes.c_int32),
                ("leaf_tc", ctypes.c_int32), ("reserved", ctypes.c_int32 * 4)]


class _Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "n_nodes", "n_leaves", "n_sums", "n_products", "n_sum_edges", "n_tasks",
        "n_cut_values", "partition_cost", "n_records", "n_global_slots", "n_smem_slots",
        "max_stack", "mufu_per_sample", "fma_per_sample", "bytes_per_sample",
        "tc_flops_per_sample")] + [
        (n, ctypes.c_int32) for n in ("path", "block_threads", "samples_per_thread", "grid",
                                      "smem_bytes", "x_in_smem")] + [
        ("prepare_ms", ctypes.c_double), ("kernel_regs", ctypes.c_int32),
        ("ctas_per_sm", ctypes.c_int32), ("mufu_exec_per_sample", ctypes.c_int64),
        ("compile_ms", ctypes.c_double), ("chunk_samples", ctypes.c_int64),
        ("layered_kernel", ctypes.c_int32), ("tc_passes", ctypes.c_int32),
        ("value_space", ctypes.c_int32), ("certified", ctypes.c_int32),
        ("cert_err", ctypes.c_double), ("leaf_tc", ctypes.c_int32)]


_lib = None


def load_library(path: str | None = None):
    """Load libspnb.so (built by ``build.build()``).  Raises if missing."""
    global _lib
    if _lib is not None:
        return _lib
    path = path or os.environ.get("SPNB_LIB") or _LIB_PATH  # SPNB_LIB: variant builds (experiments)
    if not os.path.exists(path):
        raise ImportError(f"libspnb.so not built ({path}); run __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    P, I32, I64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    lib.spn_last_error.restype = ctypes.c_char_p
    lib.spn_default_options.argtypes = [P]
    lib.spn_load_graph.argtypes = [P, I64, P, P, I64, P, I64, P, I32, I32, P]
    lib.spn_prepare.argtypes = [P, P, P]
    for fn in (lib.spn_infer_joint, lib.spn_infer_marginal):
        fn.argtypes = [P, P, I64, I64, P, P, P]
    for fn in (lib.spn_infer_joint_host, lib.spn_infer_marginal_host):
        fn.argtypes = [P, P, I64, I64, P, P]
    lib.spn_plan_info.argtypes = [P, P]
    lib.spn_free.argtypes = [P]
    lib.spn_free.restype = None
    lib.spn_partition_graph.argtypes = [P, I64, P, P, P, P]
    lib.spn_build_program.argtypes = [P, I32, I32, I64, I64, P, P, P, P, P, P, P, P, P]
    lib.spn_build_layered.argtypes = [P, P, P, I64, P, P, P, P, P, P]
    lib.spn_build_layered2.argtypes = [P, P, P, I64, P, P, P, P, P, P, P, P]
    lib.spn_codegen.argtypes = [P, I32, I32, P, P, P, P, P, P, P, P, I32, ctypes.c_char_p]
    for name in ("spn_load_graph", "spn_prepare", "spn_infer_joint", "spn_infer_marginal",
                 "spn_infer_joint_host", "spn_infer_marginal_host", "spn_plan_info",
                 "spn_partition_graph", "spn_build_program", "spn_build_layered",
                 "spn_build_layered2", "spn_codegen"):
        getattr(lib, name).restype = ctypes.c_int
    _lib = lib
    return lib


def _check(rc: int):
    if rc != 0:
        raise SPNError(rc, load_library().spn_last_error().decode())


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


class Graph:
    """A validated copy of an SPN DAG (``spn_load_graph``).  ``spn`` is any
    object with the flat arrays of ``spn_inputs.FlatSPN`` (kind, feature,
    child_begin, n_children, param_begin, n_params, children, weights,
    params, roots, n_features)."""

    def __init__(self, spn):
        lib = load_library()
        n = int(np.asarray(spn.kind).shape[0])
        nodes = np.zeros(n, dtype=NODE_DTYPE)
        nodes["kind"] = spn.kind
        nodes["feature"] = spn.feature
        nodes["child_begin"] = spn.child_begin
        nodes["param_begin"] = spn.param_begin
        nodes["n_children"] = spn.n_children
        nodes["n_params"] = spn.n_params
        ch = np.ascontiguousarray(spn.children, dtype=np.int64)
        w = np.ascontiguousarray(spn.weights, dtype=np.float64)
        prm = np.ascontiguousarray(spn.params, dtype=np.float64)
        roots = np.ascontiguousarray(spn.roots, dtype=np.int64)
        h = ctypes.c_void_p()
        _check(lib.spn_load_graph(_ptr(nodes), n, _ptr(ch), _ptr(w), ch.shape[0], _ptr(prm),
                                  prm.shape[0], _ptr(roots), roots.shape[0],
                                  int(spn.n_features), ctypes.byref(h)))
        self._h = h
        self.n_nodes = n
        self.n_roots = int(roots.shape[0])
        self.n_features = int(spn.n_features)

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None):
            load_library().spn_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Plan:
    """A prepared inference plan on one GPU (``spn_prepare``)."""

    def __init__(self, graph: Graph, device: int | None = None, block_threads: int = 0,
                 samples_per_thread: int = 0, max_task_nodes: int = 0,
                 layered_path: int = 0, tc_precision: int = 0, ctas_per_sm: int = 0,
                 compiled_path: int = 0, layered_kernel: int = 0, value_space: int = 0,
                 leaf_tc: int = 0):
        lib = load_library()
        opt = _Options()
        lib.spn_default_options(ctypes.byref(opt))
        if device is None:
            import torch
            device = torch.cuda.current_device()
        opt.device = int(device)
        opt.block_threads = block_threads
        opt.samples_per_thread = samples_per_thread
        opt.max_task_nodes = max_task_nodes
        opt.layered_path = layered_path
        opt.tc_precision = tc_precision
        opt.ctas_per_sm = ctas_per_sm
        opt.compiled_path = compiled_path
        opt.layered_kernel = layered_kernel
        opt.value_space = value_space
        opt.leaf_tc = leaf_tc
        h = ctypes.c_void_p()
        _check(lib.spn_prepare(graph.handle, ctypes.byref(opt), ctypes.byref(h)))
        self._h = h
        self.device = int(device)
        self.n_roots = graph.n_roots
        self.n_features = graph.n_features

    def info(self) -> dict:
        s = _Stats()
        _check(load_library().spn_plan_info(self._h, ctypes.byref(s)))
        return {n: getattr(s, n) for n, _ in _Stats._fields_}

    def infer(self, x, marginal: bool = False, out=None, argmax=None, want_argmax=True,
              stream=None):
        """x: CUDA float32 tensor [N, >=F] with unit stride in the feature
        dimension.  Returns (logp [N, R] float32, argmax [N] int32 or None).
        Asynchronous on ``stream`` (default: torch's current stream)."""
        import torch
        if not (x.is_cuda and x.dtype == torch.float32 and x.dim() == 2 and x.stride(1) == 1):
            raise ValueError("x must be a CUDA float32 [N, F] tensor with unit feature stride")
        if x.shape[1] < self.n_features:
            raise ValueError(f"x has {x.shape[1]} features, the SPN needs {self.n_features}")
        if x.device.index != self.device:
            raise ValueError(f"x is on cuda:{x.device.index}, the plan on cuda:{self.device}")
        N = x.shape[0]
        if out is None:
            out = torch.empty((N, self.n_roots), dtype=torch.float32, device=x.device)
        elif not (out.is_cuda and out.device.index == self.device and out.dtype == torch.float32
                  and tuple(out.shape) == (N, self.n_roots) and out.is_contiguous()):
            raise ValueError(f"out must be a contiguous float32 [{N}, {self.n_roots}] tensor "
                             f"on cuda:{self.device}")
        if argmax is None and want_argmax:
            argmax = torch.empty((N,), dtype=torch.int32, device=x.device)
        elif argmax is not None and not (
                argmax.is_cuda and argmax.device.index == self.device
                and argmax.dtype == torch.int32 and tuple(argmax.shape) == (N,)
                and argmax.is_contiguous()):
            raise ValueError(f"argmax must be a contiguous int32 [{N}] tensor on cuda:{self.device}")
        st = stream if stream is not None else torch.cuda.current_stream(x.device)
        fn = load_library().spn_infer_marginal if marginal else load_library().spn_infer_joint
        _check(fn(self._h, ctypes.c_void_p(x.data_ptr()), N, x.stride(0),
                  ctypes.c_void_p(out.data_ptr()),
                  ctypes.c_void_p(argmax.data_ptr()) if argmax is not None else None,
                  ctypes.c_void_p(st.cuda_stream)))
        return out, argmax

    def infer_host(self, x, marginal: bool = False, out=None, argmax=None, want_argmax=True):
        """End-to-end inference from HOST memory (numpy or CPU torch tensor,
        ideally pinned); copies are overlapped with compute inside the
        library.  Synchronous."""
        xa = x.numpy() if hasattr(x, "numpy") and not isinstance(x, np.ndarray) else x
        if not (isinstance(xa, np.ndarray) and xa.dtype == np.float32 and xa.ndim == 2
                and xa.strides[1] == 4):
            raise ValueError("x must be a float32 [N, F] host array with unit feature stride")
        if xa.shape[1] < self.n_features:
            raise ValueError(f"x has {xa.shape[1]} features, the SPN needs {self.n_features}")
        N = xa.shape[0]
        if out is None:
            out = np.empty((N, self.n_roots), dtype=np.float32)
        if argmax is None and want_argmax:
            argmax = np.empty((N,), dtype=np.int32)
        outa = out.numpy() if hasattr(out, "numpy") and not isinstance(out, np.ndarray) else out
        ama = argmax.numpy() if (argmax is not None and hasattr(argmax, "numpy")
                                 and not isinstance(argmax, np.ndarray)) else argmax
        if not (isinstance(outa, np.ndarray) and outa.dtype == np.float32
                and outa.shape == (N, self.n_roots) and outa.flags["C_CONTIGUOUS"]):
            raise ValueError(f"out must be a contiguous float32 [{N}, {self.n_roots}] host array")
        if ama is not None and not (isinstance(ama, np.ndarray) and ama.dtype == np.int32
                                    and ama.shape == (N,) and ama.flags["C_CONTIGUOUS"]):
            raise ValueError(f"argmax must be a contiguous int32 [{N}] host array")
        fn = (load_library().spn_infer_marginal_host if marginal
              else load_library().spn_infer_joint_host)
        _check(fn(self._h, _ptr(xa), N, xa.strides[0] // 4, _ptr(outa),
                  _ptr(ama) if ama is not None else None))
        return out, argmax

    def close(self):
        if getattr(self, "_h", None):
            load_library().spn_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def partition_graph(graph: Graph, max_task_ops: int):
    """Host-only: task id per original node (-1 leaves / removed nodes),
    n_tasks, cost, cut_values (``spn_partition_graph``)."""
    lib = load_library()
    t = np.empty(graph.n_nodes, dtype=np.int32)
    nt = ctypes.c_int32()
    cost = ctypes.c_int64()
    cut = ctypes.c_int64()
    _check(lib.spn_partition_graph(graph.handle, int(max_task_ops), _ptr(t), ctypes.byref(nt),
                                   ctypes.byref(cost), ctypes.byref(cut)))
    return t, int(nt.value), int(cost.value), int(cut.value)


def build_program(graph: Graph, samples_per_thread: int = 4, x_in_smem: bool = True,
                  max_task_ops: int = -1, smem_slot_cap: int = 0):
    """Host-only: the node program the preparer generates (``spn_build_program``).
    Returns dict(records, task_off, tables, edges, n_sslots, n_gslots, max_stack)."""
    lib = load_library()
    nr, nt, ntab, ne = (ctypes.c_int64() for _ in range(4))
    slots = np.zeros(3, dtype=np.int64)
    args = (graph.handle, samples_per_thread, int(bool(x_in_smem)), int(max_task_ops),
            int(smem_slot_cap))
    _check(lib.spn_build_program(*args, None, ctypes.byref(nr), None, ctypes.byref(nt), None,
                                 ctypes.byref(ntab), None, ctypes.byref(ne), _ptr(slots)))
    rec = np.zeros(nr.value, dtype=REC_DTYPE)
    toff = np.zeros(nt.value + 1, dtype=np.int64)
    tab = np.zeros(ntab.value, dtype=np.float32)
    edg = np.zeros(ne.value, dtype=EDGE_DTYPE)
    _check(lib.spn_build_program(*args, _ptr(rec), ctypes.byref(nr), _ptr(toff),
                                 ctypes.byref(nt), _ptr(tab), ctypes.byref(ntab), _ptr(edg),
                                 ctypes.byref(ne), _ptr(slots)))
    return {"records": rec, "task_off": toff, "tables": tab, "edges": edg,
            "n_sslots": int(slots[0]), "n_gslots": int(slots[1]), "max_stack": int(slots[2])}


def build_layered(graph: Graph):
    """Host-only: the layered (RAT-SPN) tensor-core plan (``spn_build_layered``).
    Returns None (and the reason) if the DAG is not a layered region graph."""
    lib = load_library()
    ok = ctypes.c_int32()
    why = ctypes.create_string_buffer(256)
    sizes = np.zeros(7, dtype=np.int64)
    _check(lib.spn_build_layered(graph.handle, ctypes.byref(ok), why, 256, _ptr(sizes),
                                 None, None, None, None, None))
    if not ok.value:
        return None, why.value.decode()
    assert sizes[6] == LSTEP_DTYPE.itemsize, (sizes[6], LSTEP_DTYPE.itemsize)
    steps = np.zeros(sizes[0], dtype=LSTEP_DTYPE)
    vars_ = np.zeros(sizes[1], dtype=np.int32)
    fp = np.zeros(sizes[2], dtype=np.float32)
    w = np.zeros(sizes[3] // 2, dtype=np.float16)
    rm = np.zeros(sizes[4], dtype=np.int32)
    _check(lib.spn_build_layered(graph.handle, ctypes.byref(ok), why, 256, _ptr(sizes),
                                 _ptr(steps), _ptr(vars_), _ptr(fp), _ptr(w), _ptr(rm)))
    return {"steps": steps, "vars": vars_, "fparams": fp, "wimg": w, "root_map": rm,
            "smem_floats": int(sizes[5])}, ""


R2STEP_DTYPE = np.dtype([(n, "<i4") for n in ("type", "root", "n_out", "na", "nb", "kpad",
                                              "n_groups", "spg_a", "ncol_a", "spg_b", "ncol_b",
                                              "slot_a", "slot_b", "slot_out", "n_vars", "pad_")] +
                        [(n, "<i8") for n in ("vars_off", "blk_off", "blk_floats", "w_off",
                                              "wbytes_a", "wbytes_b")])


def build_layered2(graph: Graph, leaf_tc: bool = False):
    """Host-only: the v2 layered kernel's plan (``spn_build_layered2_ex``;
    leaf_tc: the tensor-core leaf variant).  Returns (plan dict, "") or
    (None, reason)."""
    lib = load_library()
    ok = ctypes.c_int32()
    why = ctypes.create_string_buffer(256)
    sizes = np.zeros(6, dtype=np.int64)
    dims = np.zeros(14, dtype=np.int32)
    err = ctypes.c_double()
    lt = 1 if leaf_tc else 0
    _check(lib.spn_build_layered2_ex(graph.handle, lt, ctypes.byref(ok), why, 256, _ptr(sizes),
                                     _ptr(dims), None, None, None, None, None, ctypes.byref(err)))
    if not ok.value:
        return None, why.value.decode()
    assert sizes[5] == R2STEP_DTYPE.itemsize, (sizes[5], R2STEP_DTYPE.itemsize)
    steps = np.zeros(sizes[0], dtype=R2STEP_DTYPE)
    vars_ = np.zeros(sizes[1], dtype=np.int32)
    fp = np.zeros(sizes[2], dtype=np.float32)
    w = np.zeros(sizes[3] // 2, dtype=np.float16)
    rm = np.zeros(sizes[4], dtype=np.int32)
    _check(lib.spn_build_layered2_ex(graph.handle, lt, ctypes.byref(ok), why, 256, _ptr(sizes),
                                     _ptr(dims), _ptr(steps), _ptr(vars_), _ptr(fp), _ptr(w),
                                     _ptr(rm), None))
    keys = ("F", "C", "I", "S", "D", "gcols", "kpad_bot", "kpad_up", "max_wgroup", "max_vars",
            "max_blk", "lvp", "kl_j", "kl_m")
    return {"steps": steps, "vars": vars_, "fparams": fp, "wimg": w, "root_map": rm,
            "tc_err_1pass": float(err.value), "leaf_tc": bool(leaf_tc),
            **{k: int(v) for k, v in zip(keys, dims)}}, ""


def codegen(graph: Graph, task: int = 0, lang: str = "cpp", compile: bool = False,
            arch: str = "100a", space: int = 0):
    """Host-only: the compiled path's generated code for one task
    (``spn_codegen``): lang "ptx" (what the library assembles) or "cpp" (the
    same IR as host C++, for CPU checks).  Returns dict(source, name, roots,
    tables, n_tasks).  compile=True also assembles the PTX for sm_<arch>
    with nvJitLink (raises SPNError on failure)."""
    lg = {"cpp": 0, "ptx": 1}[lang] | (int(space) << 8)   # space: 0 auto, 1 log2, 2 linear
    lib = load_library()
    sl, nt = ctypes.c_int64(), ctypes.c_int64()
    nr, ntask = ctypes.c_int32(), ctypes.c_int32()
    _check(lib.spn_codegen(graph.handle, int(task), lg, None, ctypes.byref(sl), None, None,
                           ctypes.byref(nr), None, ctypes.byref(nt), ctypes.byref(ntask), 0,
                           arch.encode()))
    src = ctypes.create_string_buffer(sl.value)
    name = ctypes.create_string_buffer(64)
    roots = np.zeros(max(1, nr.value), dtype=np.int32)
    tab = np.zeros(max(1, nt.value), dtype=np.float32)
    _check(lib.spn_codegen(graph.handle, int(task), lg, src, ctypes.byref(sl), name, _ptr(roots),
                           ctypes.byref(nr), _ptr(tab), ctypes.byref(nt), ctypes.byref(ntask),
                           int(bool(compile)), arch.encode()))
    return {"source": src.value.decode(), "name": name.value.decode(),
            "roots": roots[:nr.value].copy(), "tables": tab[:nt.value].copy(),
            "n_tasks": int(ntask.value)}
