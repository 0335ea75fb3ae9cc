"""Thin ctypes binding of libfop.so (include/fop.h) — argument marshalling only.

Every step of the fused operator runs in libfop: validation, the Algorithm-2
planner, kernel generation/compilation (NVRTC, sm_100a) and the kernels.
PyTorch only supplies device memory and the CUDA stream.  There is no CPU or
PyTorch fallback: if libfop.so is missing, importing this module fails.

    op = FusedOp(desc)                 # desc: the dict form of workloads/
    op.run({"x": x, "y": y, ...})      # torch CUDA tensors, current stream
"""
import ctypes as C
import os

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libfop.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with "
                      "`python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build` "
                      "(there is no fallback path)")
_lib = C.CDLL(LIB_PATH)

MAX_RANK, MAX_LOOPS, MAX_TENSORS, MAX_STMTS = 8, 8, 16, 8
MAX_ACC, MAX_NODES, MAX_FIN, MAX_LAUNCH, MAX_SCEN, MAX_DEPS = 8, 48, 8, 8, 8, 16
MAX_PEERS = 8

DTYPE = {"f32": 0, "f16": 1, "bf16": 2, "i32": 3}
ROLE = {"in": 1, "out": 2, "inout": 3, "temp": 4}
KIND = {"assign": 0, "reduce": 1}
REDOP = {"sum": 0, "max": 1}
OPC = {"load": 0, "const": 1, "acc": 2, "add": 3, "sub": 4, "mul": 5, "div": 6, "max": 7,
       "min": 8, "neg": 9, "abs": 10, "sqrt": 11, "relu": 12, "exp": 13, "log": 14,
       "tanh": 15, "sigmoid": 16, "gelu_tanh": 17, "gelu_erf": 18, "cast": 19}
CLASS_NAMES = {0: "ew", 1: "transpose", 2: "row_reduce", 3: "col_reduce"}
STATUS = {0: "FOP_OK", 1: "FOP_E_INVALID", 2: "FOP_E_UNSUPPORTED", 3: "FOP_E_ALIGN",
          4: "FOP_E_CUDA", 5: "FOP_E_NOMEM", 6: "FOP_E_JIT"}
ORDER = {"paper": 0, "memory": 1}


class Tensor(C.Structure):
    _fields_ = [("rank", C.c_int32), ("dtype", C.c_int32), ("role", C.c_int32), ("_pad", C.c_int32),
                ("shape", C.c_int64 * MAX_RANK), ("stride", C.c_int64 * MAX_RANK)]


class Access(C.Structure):
    _fields_ = [("tensor", C.c_int32), ("loop", C.c_int32 * MAX_RANK), ("offset", C.c_int64 * MAX_RANK)]


class Node(C.Structure):
    _fields_ = [("op", C.c_int32), ("a", C.c_int32), ("b", C.c_int32), ("cvt", C.c_int32),
                ("imm", C.c_float), ("_pad", C.c_int32)]


class Stmt(C.Structure):
    _fields_ = [("kind", C.c_int32), ("reduce_op", C.c_int32), ("nloops", C.c_int32),
                ("loop", C.c_int32 * MAX_LOOPS), ("nacc", C.c_int32), ("acc", Access * MAX_ACC),
                ("nnodes", C.c_int32), ("node", Node * MAX_NODES), ("nfin", C.c_int32),
                ("fin", Node * MAX_FIN)]


class Desc(C.Structure):
    _fields_ = [("nloops", C.c_int32), ("extent", C.c_int64 * MAX_LOOPS), ("ntensors", C.c_int32),
                ("t", Tensor * MAX_TENSORS), ("nstmts", C.c_int32), ("s", Stmt * MAX_STMTS)]


class PlanOpts(C.Structure):
    _fields_ = [("w", C.c_double * 5), ("thread_limit", C.c_int32), ("max_scenarios", C.c_int32),
                ("max_vec_bytes", C.c_int32), ("readings", C.c_int32), ("force_width", C.c_int32),
                ("coalesce_order", C.c_int32), ("sm_count", C.c_int32), ("jit", C.c_int32),
                ("autotune", C.c_int32), ("peer_world", C.c_int32), ("peer_loop", C.c_int32),
                ("peer_timeout_ms", C.c_int32), ("variant", C.c_int32)]


class LaunchInfo(C.Structure):
    _fields_ = [("kernel_class", C.c_int32), ("main_stmt", C.c_int32), ("stmt_mask", C.c_uint32),
                ("vec_loop", C.c_int32), ("width", C.c_int32), ("read_loop", C.c_int32),
                ("read_width", C.c_int32), ("coal_loop", C.c_int32), ("grid", C.c_int64),
                ("block", C.c_int32), ("nseq", C.c_int32), ("seq", C.c_int32 * MAX_LOOPS),
                ("scen_pick", C.c_int32), ("fallback", C.c_int32), ("peer_exchange", C.c_int32),
                ("nvariants", C.c_int32)]


class PlanInfo(C.Structure):
    _fields_ = [("nstmts", C.c_int32), ("nscen", C.c_int32 * MAX_STMTS),
                ("scen_len", (C.c_int32 * MAX_SCEN) * MAX_STMTS),
                ("scenario", ((C.c_int32 * 3) * MAX_SCEN) * MAX_STMTS),
                ("inner_score", (C.c_double * MAX_LOOPS) * MAX_STMTS),
                ("nlaunch", C.c_int32), ("launch", LaunchInfo * MAX_LAUNCH),
                ("workspace_bytes", C.c_size_t), ("ndeps", C.c_int32 * MAX_STMTS),
                ("dep", ((C.c_int64 * MAX_LOOPS) * MAX_DEPS) * MAX_STMTS),
                ("dep_anti", (C.c_int32 * MAX_DEPS) * MAX_STMTS)]


_lib.fop_abi_version.restype = C.c_int
ABI_VERSION = 4   # the struct layouts above mirror include/fop.h at this version
if _lib.fop_abi_version() != ABI_VERSION:
    raise ImportError(f"{LIB_PATH}: ABI version {_lib.fop_abi_version()} != binding {ABI_VERSION}; rebuild "
                      "with python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build")
_lib.fop_plan_opts_default.argtypes = [C.POINTER(PlanOpts)]
_lib.fop_plan.argtypes = [C.POINTER(Desc), C.POINTER(PlanOpts), C.POINTER(C.c_void_p)]
_lib.fop_plan.restype = C.c_int
_lib.fop_plan_info_get.argtypes = [C.c_void_p, C.POINTER(PlanInfo)]
_lib.fop_plan_info_get.restype = C.c_int
_lib.fop_plan_workspace_bytes.argtypes = [C.c_void_p]
_lib.fop_plan_workspace_bytes.restype = C.c_size_t
_lib.fop_plan_source.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_char_p)]
_lib.fop_plan_source.restype = C.c_int
_lib.fop_plan_cubin.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_void_p), C.POINTER(C.c_size_t)]
_lib.fop_plan_cubin.restype = C.c_int
_lib.fop_run.argtypes = [C.c_void_p, C.POINTER(C.c_void_p), C.c_int32, C.c_void_p, C.c_void_p]
_lib.fop_run.restype = C.c_int
_lib.fop_run_host.argtypes = [C.c_void_p, C.POINTER(C.c_void_p), C.POINTER(C.c_void_p), C.c_int32,
                              C.c_void_p, C.c_void_p]
_lib.fop_run_host.restype = C.c_int
_lib.fop_run_host_many.argtypes = [C.POINTER(C.c_void_p), C.POINTER(C.POINTER(C.c_void_p)),
                                   C.POINTER(C.POINTER(C.c_void_p)), C.POINTER(C.c_int32), C.POINTER(C.c_void_p),
                                   C.c_int32, C.c_void_p]
_lib.fop_run_host_many.restype = C.c_int
_lib.fop_plan_selected.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_char_p), C.POINTER(C.c_int64),
                                   C.POINTER(C.c_int32)]
_lib.fop_plan_selected.restype = C.c_int
_lib.fop_plan_destroy.argtypes = [C.c_void_p]


class IpcHandle(C.Structure):
    _fields_ = [("bytes", C.c_ubyte * 64)]


class PeerGroupC(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("buf", C.c_void_p * MAX_PEERS)]


_lib.fop_run_many.argtypes = [C.POINTER(C.c_void_p), C.POINTER(C.POINTER(C.c_void_p)), C.POINTER(C.c_int32),
                              C.POINTER(C.c_void_p), C.c_int32, C.c_void_p]
_lib.fop_run_many.restype = C.c_int
_lib.fop_plan_peer_bytes.argtypes = [C.c_void_p]
_lib.fop_plan_peer_bytes.restype = C.c_size_t
_lib.fop_run_peer.argtypes = [C.c_void_p, C.POINTER(C.c_void_p), C.c_int32, C.c_void_p, C.POINTER(PeerGroupC),
                              C.c_void_p]
_lib.fop_run_peer.restype = C.c_int
_lib.fop_peer_alloc.argtypes = [C.c_size_t, C.POINTER(C.c_void_p), C.POINTER(IpcHandle)]
_lib.fop_peer_alloc.restype = C.c_int
_lib.fop_peer_free.argtypes = [C.c_void_p]
_lib.fop_peer_free.restype = C.c_int
_lib.fop_peer_open.argtypes = [C.POINTER(IpcHandle), C.POINTER(C.c_void_p)]
_lib.fop_peer_open.restype = C.c_int
_lib.fop_peer_close.argtypes = [C.c_void_p]
_lib.fop_peer_close.restype = C.c_int
_lib.fop_status_str.restype = C.c_char_p
_lib.fop_last_error.restype = C.c_char_p

ABI_SYMBOLS = ["fop_abi_version", "fop_plan_opts_default", "fop_plan", "fop_plan_info_get",
               "fop_plan_workspace_bytes", "fop_plan_source", "fop_plan_cubin", "fop_run",
               "fop_run_host", "fop_run_host_many", "fop_plan_selected", "fop_plan_destroy", "fop_status_str",
               "fop_last_error", "fop_run_many", "fop_plan_peer_bytes", "fop_run_peer", "fop_peer_alloc", "fop_peer_free",
               "fop_peer_open", "fop_peer_close"]


class FopError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = STATUS.get(status, status)


def _check(rc):
    if rc != 0:
        raise FopError(rc, _lib.fop_last_error().decode(errors="replace"))


def _strides(t):
    if t.get("strides"):
        return list(t["strides"])
    st, acc = [], 1
    for s in reversed(t["shape"]):
        st.append(acc)
        acc *= s
    return list(reversed(st))


def span_elems(t):
    if any(s == 0 for s in t["shape"]):
        return 0
    return 1 + sum((s - 1) * k for s, k in zip(t["shape"], _strides(t)))


ESIZE = {"f32": 4, "f16": 2, "bf16": 2, "i32": 4}


def _torch_dtype(name):
    import torch
    return {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16, "i32": torch.int32}[name]


def marshal(desc):
    """dict form (workloads/) -> fop_desc."""
    d = Desc()
    loops = list(desc["loops"].keys())
    lid = {n: i for i, n in enumerate(loops)}
    names = list(desc["tensors"].keys())
    tid = {n: i for i, n in enumerate(names)}
    d.nloops = len(loops)
    for i, n in enumerate(loops):
        d.extent[i] = int(desc["loops"][n])
    d.ntensors = len(names)
    for i, n in enumerate(names):
        t = desc["tensors"][n]
        d.t[i].rank = len(t["shape"])
        d.t[i].dtype = DTYPE[t["dtype"]]
        d.t[i].role = ROLE[t["role"]]
        for r, (s, k) in enumerate(zip(t["shape"], _strides(t))):
            d.t[i].shape[r] = int(s)
            d.t[i].stride[r] = int(k)

    def access(a, acc):
        name, index = acc
        a.tensor = tid[name]
        for r in range(MAX_RANK):
            a.loop[r] = -1
            a.offset[r] = 0
        for r, e in enumerate(index):
            if isinstance(e, str):
                a.loop[r] = lid[e]
            elif isinstance(e, (tuple, list)):
                a.loop[r] = lid[e[0]]
                a.offset[r] = int(e[1])
            else:
                a.offset[r] = int(e)

    def node(n, spec):
        n.op = OPC[spec[0]]
        n.a = n.b = -1
        n.cvt = 0
        n.imm = 0.0
        if spec[0] == "load":
            n.a = int(spec[1]) + 1          # access 0 is the write
        elif spec[0] == "const":
            n.imm = float(spec[1])
        elif spec[0] == "acc":
            pass
        elif spec[0] == "cast":
            n.a = int(spec[1])
            n.cvt = DTYPE[spec[2]]
        elif spec[0] in ("add", "sub", "mul", "div", "max", "min"):
            n.a, n.b = int(spec[1]), int(spec[2])
        else:
            n.a = int(spec[1])

    d.nstmts = len(desc["stmts"])
    for si, s in enumerate(desc["stmts"]):
        st = d.s[si]
        st.kind = KIND[s["kind"]]
        st.reduce_op = REDOP[s.get("op", "sum")]
        st.nloops = len(s["loops"])
        for k, l in enumerate(s["loops"]):
            st.loop[k] = lid[l]
        st.nacc = 1 + len(s["reads"])
        access(st.acc[0], s["write"])
        for k, r in enumerate(s["reads"]):
            access(st.acc[k + 1], r)
        st.nnodes = len(s["expr"])
        for k, e in enumerate(s["expr"]):
            node(st.node[k], e)
        fin = s.get("finalize") or []
        st.nfin = len(fin)
        for k, e in enumerate(fin):
            node(st.fin[k], e)
    return d


def default_opts(**kw):
    o = PlanOpts()
    _lib.fop_plan_opts_default(C.byref(o))
    for k, v in kw.items():
        if k == "w":
            for i, x in enumerate(v):
                o.w[i] = float(x)
        elif k == "coalesce_order":
            o.coalesce_order = ORDER[v] if isinstance(v, str) else int(v)
        else:
            setattr(o, k, int(v))
    return o


class FusedOp:
    """A planned (and compiled) fused operator: fop_plan + fop_run."""

    def __init__(self, desc, **opts):
        self.desc = desc
        self.names = list(desc["tensors"].keys())
        self.loops = list(desc["loops"].keys())
        self._c_desc = marshal(desc)
        if isinstance(opts.get("peer_loop"), str):
            opts["peer_loop"] = self.loops.index(opts["peer_loop"])
        self._opts = default_opts(**opts)
        h = C.c_void_p()
        _check(_lib.fop_plan(C.byref(self._c_desc), C.byref(self._opts), C.byref(h)))
        self._h = h
        self._ws = {}

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            try:
                _lib.fop_plan_destroy(h)
            except Exception:       # interpreter shutdown
                pass
            self._h = None

    # ------------------------------------------------------------ planner view
    def info(self):
        pi = PlanInfo()
        _check(_lib.fop_plan_info_get(self._h, C.byref(pi)))
        ln = lambda i: self.loops[i] if i >= 0 else None  # noqa: E731
        stmts = []
        for s in range(pi.nstmts):
            sl = self.desc["stmts"][s]["loops"]
            stmts.append({
                "scenarios": [[ln(pi.scenario[s][k][q]) for q in range(pi.scen_len[s][k])]
                              for k in range(pi.nscen[s])],
                "inner_score": {sl[k]: pi.inner_score[s][k] for k in range(len(sl))},
                # uniform self-dependences (distance by loop name, lexicographically positive)
                "deps": [{"dist": {self.loops[l]: pi.dep[s][k][l] for l in range(len(self.loops))
                                   if pi.dep[s][k][l] != 0},
                          "anti": bool(pi.dep_anti[s][k])} for k in range(pi.ndeps[s])],
            })
        launches = []
        for i in range(pi.nlaunch):
            li = pi.launch[i]
            launches.append({"class": CLASS_NAMES[li.kernel_class], "main_stmt": li.main_stmt,
                             "stmts": [s for s in range(8) if li.stmt_mask >> s & 1],
                             "vec_loop": ln(li.vec_loop), "width": li.width,
                             "read_loop": ln(li.read_loop), "read_width": li.read_width,
                             "coal_loop": ln(li.coal_loop), "grid": li.grid, "block": li.block,
                             "seq": [ln(li.seq[q]) for q in range(li.nseq)],
                             "scen_pick": li.scen_pick, "fallback": li.fallback,
                             "peer_exchange": bool(li.peer_exchange), "nvariants": li.nvariants})
        return {"stmts": stmts, "launches": launches, "workspace_bytes": pi.workspace_bytes}

    @property
    def nlaunch(self):
        return len(self.info()["launches"])

    def source(self, i=0, narrow=False):
        """CUDA source of launch i (narrow=True: its misaligned-pointer variant)."""
        s = C.c_char_p()
        _check(_lib.fop_plan_source(self._h, -1 - i if narrow else i, C.byref(s)))
        return s.value.decode()

    def cubin(self, i=0):
        p, n = C.c_void_p(), C.c_size_t()
        _check(_lib.fop_plan_cubin(self._h, i, C.byref(p), C.byref(n)))
        return C.string_at(p, n.value)

    def selected(self, i=0):
        """(kernel name, grid, block) fop_run launches for launch i on the current context."""
        nm, g, b = C.c_char_p(), C.c_int64(), C.c_int32()
        _check(_lib.fop_plan_selected(self._h, i, C.byref(nm), C.byref(g), C.byref(b)))
        return nm.value.decode(), g.value, b.value

    @property
    def workspace_bytes(self):
        return _lib.fop_plan_workspace_bytes(self._h)

    @property
    def peer_bytes(self):
        """Exchange-buffer size of a plan with opts.peer_world >= 1 (else 0)."""
        return _lib.fop_plan_peer_bytes(self._h)

    # ------------------------------------------------------------ execution
    def _workspace(self, device, stream):
        """The cached zero-filled workspace for (device, stream).  Runs of one plan on
        DIFFERENT streams may overlap, and a workspace holds per-run state (COL_REDUCE
        partial sums and arrival counters, TEMP tensors), so each stream gets its own."""
        import torch
        n = self.workspace_bytes
        if n == 0:
            return None
        key = (str(device), int(stream.cuda_stream))
        if key not in self._ws:
            self._ws[key] = torch.zeros(n, dtype=torch.uint8, device=device)  # zero-filled (fop.h)
        return self._ws[key]

    def _check_tensor(self, n, t, where):
        """A buffer handed to the C ABI must hold the descriptor's dtype and every
        element the descriptor addresses from its base pointer (the library sees
        pointers only, so this is the last place a short buffer can be caught)."""
        chk = self.__dict__.get("_chk")
        if chk is None:   # per tensor: torch dtype and bytes addressed from the base pointer
            chk = self._chk = {m: (_torch_dtype(sp["dtype"]), span_elems(sp) * ESIZE[sp["dtype"]])
                               for m, sp in self.desc["tensors"].items()}
        want, need = chk[n]
        if t.dtype is not want:
            if not hasattr(t, "untyped_storage"):
                raise TypeError(f"tensor {n!r}: expected a torch.Tensor, got {type(t).__name__}")
            raise TypeError(f"tensor {n!r}: dtype {t.dtype}, the descriptor says "
                            f"{self.desc['tensors'][n]['dtype']} ({want})")
        if t.is_cuda != (where == "cuda"):
            raise ValueError(f"tensor {n!r} is on {t.device}, expected a {'CUDA' if where == 'cuda' else 'host'} tensor")
        # the library addresses memory from data_ptr() with the DESCRIPTOR's strides: a strided
        # view (x.t(), x[:, :768], an expand) would silently read or write other elements
        if not t.is_contiguous():
            sp = self.desc["tensors"][n]
            st = _strides(sp)
            if t.dim() != len(sp["shape"]) or any(a != b for a, b, e in zip(t.stride(), st, sp["shape"]) if e > 1):
                raise ValueError(f"tensor {n!r}: a non-contiguous view (strides {tuple(t.stride())}) whose strides "
                                 f"differ from the descriptor's {tuple(st)}; pass .contiguous() or describe its strides")
        have = t.untyped_storage().nbytes() - t.storage_offset() * t.element_size()
        if need > have:
            raise ValueError(f"tensor {n!r}: the descriptor addresses {need} bytes from its base pointer, "
                             f"the buffer holds {have}")

    def _ptrs(self, tensors):
        arr = (C.c_void_p * len(self.names))()
        dev = None
        for i, n in enumerate(self.names):
            t = tensors.get(n)
            if t is None:
                if self.desc["tensors"][n]["role"] != "temp":
                    raise ValueError(f"tensor {n!r} missing")
                arr[i] = None
                continue
            self._check_tensor(n, t, "cuda")
            if dev is not None and t.device != dev:
                raise ValueError(f"tensor {n!r} is on {t.device}, the others on {dev}")
            arr[i] = t.data_ptr()
            dev = t.device
        return arr, dev

    def _check_workspace(self, ws, dev):
        if ws is not None and self.workspace_bytes:
            have = ws.untyped_storage().nbytes() - ws.storage_offset() * ws.element_size()
            if have < self.workspace_bytes or ws.device != dev:
                raise ValueError(f"workspace: need {self.workspace_bytes} bytes on {dev}, got {have} on {ws.device}")

    def run(self, tensors, workspace=None, stream=None, peers=None):
        """Enqueue the fused operator on `stream` (default: torch's current stream).
        peers: a PeerGroup for plans with a cross-GPU exchange (fop_run_peer)."""
        import torch
        arr, dev = self._ptrs(tensors)
        if stream is None:
            stream = torch.cuda.current_stream(dev)
        ws = workspace if workspace is not None else self._workspace(dev, stream)
        self._check_workspace(ws, dev)
        if peers is not None:
            _check(_lib.fop_run_peer(self._h, arr, len(self.names), None if ws is None else ws.data_ptr(),
                                     C.byref(peers.c), stream.cuda_stream))
            return
        _check(_lib.fop_run(self._h, arr, len(self.names),
                            None if ws is None else ws.data_ptr(), stream.cuda_stream))

    def run_host(self, host, device_tensors, workspace=None, stream=None):
        """End to end: H2D copies of inputs from pinned `host`, run, D2H of outputs."""
        import torch
        arr, dev = self._ptrs(device_tensors)
        harr = self._host_ptrs(host)
        if stream is None:
            stream = torch.cuda.current_stream(dev)
        ws = workspace if workspace is not None else self._workspace(dev, stream)
        self._check_workspace(ws, dev)
        _check(_lib.fop_run_host(self._h, harr, arr, len(self.names),
                                 None if ws is None else ws.data_ptr(), stream.cuda_stream))

    def _host_ptrs(self, host):
        harr = (C.c_void_p * len(self.names))()
        for i, n in enumerate(self.names):
            h = host.get(n)
            if h is not None:
                self._check_tensor(n, h, "host")
            harr[i] = None if h is None else h.data_ptr()
        return harr


def run_host_many(items, stream=None):
    """End to end for independent operators with pipelined copies
    (fop_run_host_many): `items` is a list of (FusedOp, host tensors,
    device tensors[, workspace]); a tensor missing from `host` is not copied."""
    import torch
    n = len(items)
    plans = (C.c_void_p * n)()
    hp = (C.POINTER(C.c_void_p) * n)()
    dp = (C.POINTER(C.c_void_p) * n)()
    np_ = (C.c_int32 * n)()
    ws = (C.c_void_p * n)()
    keep = []
    dev = None
    for it in items:
        dev = dev or it[0]._ptrs(it[2])[1]
    if stream is None:
        stream = torch.cuda.current_stream(dev)
    for k, it in enumerate(items):
        op, host, devt = it[0], it[1], it[2]
        arr, d = op._ptrs(devt)
        harr = op._host_ptrs(host)
        w = it[3] if len(it) > 3 and it[3] is not None else op._workspace(d, stream)
        op._check_workspace(w, d)
        keep += [arr, harr]
        plans[k] = op._h
        hp[k] = C.cast(harr, C.POINTER(C.c_void_p))
        dp[k] = C.cast(arr, C.POINTER(C.c_void_p))
        np_[k] = len(op.names)
        ws[k] = None if w is None else w.data_ptr()
    _check(_lib.fop_run_host_many(plans, hp, dp, np_, ws, n, stream.cuda_stream))


# ---------------------------------------------------------------- peer groups (fop.h)
class PeerGroup:
    """fop_peer_group: this GPU's rank and every rank's exchange buffer as
    addressed from this process (device pointers as ints)."""

    def __init__(self, rank, bufs):
        if not 0 <= rank < len(bufs) <= MAX_PEERS:
            raise ValueError("rank/world out of range")
        self.rank, self.world = rank, len(bufs)
        self.bufs = list(bufs)
        self.c = PeerGroupC()
        self.c.rank, self.c.world = rank, len(bufs)
        for q, b in enumerate(bufs):
            self.c.buf[q] = b


def peer_alloc(nbytes):
    """Zero-filled exchange buffer on the current device: (device pointer, 64-byte IPC handle)."""
    p, h = C.c_void_p(), IpcHandle()
    _check(_lib.fop_peer_alloc(nbytes, C.byref(p), C.byref(h)))
    return p.value, bytes(h.bytes)


def peer_free(ptr):
    _check(_lib.fop_peer_free(ptr))


def peer_open(handle):
    """Map another process's exchange buffer (CUDA IPC; NVLink peer access)."""
    h = IpcHandle()
    C.memmove(h.bytes, bytes(handle), 64)
    p = C.c_void_p()
    _check(_lib.fop_peer_open(C.byref(h), C.byref(p)))
    return p.value


def peer_close(ptr):
    _check(_lib.fop_peer_close(ptr))


def run_many(items, stream=None):
    """fop_run_many: independent operators back to back, each plan's first
    kernel overlapping the previous one's tail (programmatic dependent
    launch).  `items` is a list of (FusedOp, device tensors[, workspace])."""
    import torch
    n = len(items)
    plans = (C.c_void_p * n)()
    dp = (C.POINTER(C.c_void_p) * n)()
    np_ = (C.c_int32 * n)()
    ws = (C.c_void_p * n)()
    keep = []
    dev = None
    for it in items:
        dev = dev or it[0]._ptrs(it[1])[1]
    if stream is None:
        stream = torch.cuda.current_stream(dev)
    for k, it in enumerate(items):
        op, devt = it[0], it[1]
        arr, d = op._ptrs(devt)
        w = it[2] if len(it) > 2 and it[2] is not None else op._workspace(d, stream)
        op._check_workspace(w, d)
        keep.append(arr)
        plans[k] = op._h
        dp[k] = C.cast(arr, C.POINTER(C.c_void_p))
        np_[k] = len(op.names)
        ws[k] = None if w is None else w.data_ptr()
    _check(_lib.fop_run_many(plans, dp, np_, ws, n, stream.cuda_stream))


def abi_version():
    return _lib.fop_abi_version()
