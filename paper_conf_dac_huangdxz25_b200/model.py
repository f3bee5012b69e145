"""Lower a model spec (the lowered layer sequence PASK receives, PAPER.md:91
Fig. 5) into a pask_graph over caller-owned device memory.

PyTorch is used only to allocate device memory and move bytes (weights,
inputs); every operator runs in libpask.so.  Device layouts: images NHWC bf16
(the fp32 NCHW input goes through the layout kernel, C padded to 8), matrices
row-major bf16, biases / LayerNorm vectors fp32, conv weights KRSC (dense) or
RSC (depthwise), linear weights [N][K].
"""
from __future__ import annotations

import ctypes as C

import numpy as np
import torch

from . import pask as P

_ACT = P.ACT


class _HostOnly:
    """Stand-in for a device tensor of a host-only graph: a fake address."""

    def __init__(self, ptr):
        self._p = ptr

    def data_ptr(self):
        return self._p


class DeviceModel:
    def __init__(self, spec, device="cuda", solutions=None, alloc=True):
        """spec: a workloads.models spec.  solutions: {layer index: kernel id}
        overriding the library's static choice s* for that layer.
        alloc=False builds the graph with placeholder device pointers (host-only
        planning / workspace sizing, no GPU needed)."""
        self.spec = spec
        self.device = device
        self.alloc = alloc
        self.solutions = solutions or {}
        self.t = {}        # name -> torch tensor (device)
        self.index = {}    # name -> pask tensor index
        self.dims = {}     # name -> (n, h, w, c) device dims
        self.kind = {}     # name -> "image" | "matrix" | "heads"
        self._tensors = []
        self._nodes = []
        self._keep = []
        self._blobs = {}      # pointer -> host array of every weight / bias / gamma / beta
        self._fake_next = self._FAKE
        self._build()

    # ------------------------------------------------------------ helpers
    def _dev(self, arr, dtype):
        host = torch.from_numpy(np.ascontiguousarray(arr)).to(dtype)
        if not self.alloc:
            t = _HostOnly(self._fake(host.numel() * host.element_size()))
        else:
            t = host.to(self.device)
        self._blobs[t.data_ptr()] = host
        self._keep.append(t)
        return t

    # placeholder addresses for host-only graphs (never dereferenced): distinct,
    # non-overlapping ranges, so the runtime's aliasing check sees what a real
    # allocation would give
    _FAKE = 1 << 40

    def _fake(self, nbytes):
        p = self._fake_next
        self._fake_next += (max(nbytes, 1) + 255) // 256 * 256
        return p

    def _ptr(self, t):
        return None if t is None else t.data_ptr()

    def _new(self, name, shape, dtype, layout, dims, kind):
        if self.alloc:
            t = torch.empty(shape, dtype=dtype, device=self.device)
            ptr = t.data_ptr()
        else:
            n = 1
            for d in (shape if shape is not None else dims):
                n *= d
            t, ptr = None, self._fake(n * (4 if dtype == torch.float32 else 2))
        self.t[name] = t
        self.dims[name] = dims
        self.kind[name] = kind
        self.index[name] = len(self._tensors)
        pd = P.F32 if dtype == torch.float32 else P.BF16
        self._tensors.append(P.Tensor(pd, layout, *dims, ptr))

    def _node(self, **kw):
        nd = P.Node()
        nd.in1 = nd.res = -1
        nd.solution = -1
        for k, v in kw.items():
            if k in ("stride", "pad", "dil"):
                getattr(nd, k)[0], getattr(nd, k)[1] = v
            else:
                setattr(nd, k, v)
        self._nodes.append(nd)
        return nd

    # ------------------------------------------------------------ lowering
    def _build(self):
        spec = self.spec
        for name, shape, dtype in spec["inputs"]:
            if dtype == "f32":
                n, c, h, w = shape
                self._new(name, (n, c, h, w), torch.float32, P.NCHW, (n, h, w, c), "image")
            else:
                s, hdim = shape
                self._new(name, (s, hdim), torch.bfloat16, P.ROWMAJOR, (1, 1, s, hdim), "matrix")
        for li, L in enumerate(spec["layers"]):
            op = L["op"]
            x = L["inputs"][0]
            xn, xh, xw, xc = self.dims[x]
            out = L["out"]
            sol = self.solutions.get(li, -1)
            if op == "layout":
                cp = L["c_pad"]
                self._new(out, (xn, xh, xw, cp), torch.bfloat16, P.NHWC, (xn, xh, xw, cp), "image")
                self._node(op=P.OP_LAYOUT, in0=self.index[x], out=self.index[out], solution=sol)
            elif op == "conv":
                w = L["w"]
                k, cg, r, s = w.shape
                groups = L["groups"]
                _, _, p, q = spec["tensors"][out]
                if groups == 1:
                    wd = np.zeros((k, r, s, xc), np.float32)        # KRSC, C padded
                    wd[..., :cg] = w.transpose(0, 2, 3, 1)
                else:
                    wd = w[:, 0].transpose(1, 2, 0)                   # RSC
                wt = self._dev(wd, torch.bfloat16)
                bt = self._dev(L["b"], torch.float32) if L["b"] is not None else None
                bptr = self._ptr(bt) if L["b"] is not None else None
                self._new(out, (xn, p, q, k), torch.bfloat16, P.NHWC, (xn, p, q, k), "image")
                self._node(op=P.OP_CONV2D, in0=self.index[x], out=self.index[out],
                           res=self.index[L["res"]] if L["res"] else -1,
                           w=self._ptr(wt), bias=bptr, k=k, r=r, s=s,
                           stride=L["stride"], pad=L["pad"], dil=L["dil"], groups=groups,
                           act=_ACT[L["act"]], solution=sol)
            elif op == "pool":
                _, _, p, q = spec["tensors"][out]
                self._new(out, (xn, p, q, xc), torch.bfloat16, P.NHWC, (xn, p, q, xc), "image")
                self._node(op=P.OP_POOL, in0=self.index[x], out=self.index[out],
                           r=L["kernel"][0], s=L["kernel"][1], stride=L["stride"], pad=L["pad"],
                           pool_mode=0 if L["mode"] == "max" else 1,
                           count_include_pad=1 if L["count_include_pad"] else 0,
                           global_pool=1 if L["global_"] else 0, solution=sol)
            elif op == "linear":
                w = L["w"]
                nout, kin = w.shape
                if self.kind[x] == "image":
                    # logical NCHW flatten of an NHWC device tensor: permute W's columns
                    lc = spec["tensors"][x][1]
                    wd = w.reshape(nout, lc, xh, xw).transpose(0, 2, 3, 1)
                    if xc != lc:
                        wd = np.concatenate([wd, np.zeros((nout, xh, xw, xc - lc), np.float32)], -1)
                    wd = wd.reshape(nout, -1)
                    m, kk = xn, xh * xw * xc
                else:
                    wd = w
                    m, kk = xw, xc
                if L["rows"] is not None:
                    m = L["rows"]
                wt = self._dev(wd, torch.bfloat16)
                bt = self._dev(L["b"], torch.float32) if L["b"] is not None else None
                bptr = self._ptr(bt) if L["b"] is not None else None
                self._new(out, (m, nout), torch.bfloat16, P.ROWMAJOR, (1, 1, m, nout), "matrix")
                self._node(op=P.OP_GEMM, in0=self.index[x], out=self.index[out],
                           res=self.index[L["res"]] if L["res"] else -1,
                           w=self._ptr(wt), bias=bptr, m=m, n=nout, kk=kk, batch=1,
                           trans_b=1, lda=kk, ldb=kk, ldc=nout, act=_ACT[L["act"]], solution=sol)
            elif op in ("softmax", "layernorm"):
                shape = tuple(self.t[x].shape) if self.alloc else None
                dims = self.dims[x]
                if self.kind[x] == "heads":
                    shp = (dims[0], dims[2], dims[3])
                elif self.kind[x] == "matrix":
                    shp = (dims[2], dims[3])
                else:
                    shp = shape
                self._new(out, shp, torch.bfloat16, P.ROWMAJOR, dims, self.kind[x])
                if op == "softmax":
                    self._node(op=P.OP_SOFTMAX, in0=self.index[x], out=self.index[out],
                               scale=L["scale"], solution=sol)
                else:
                    g = self._dev(L["gamma"], torch.float32)
                    b = self._dev(L["beta"], torch.float32)
                    self._node(op=P.OP_LAYERNORM, in0=self.index[x], out=self.index[out],
                               gamma=self._ptr(g), beta=self._ptr(b), eps=L["eps"], solution=sol)
            elif op == "qk":
                heads, dh = L["heads"], L["head_dim"]
                s_, three_h = xw, xc
                hid = three_h // 3
                self._new(out, (heads, s_, s_), torch.bfloat16, P.ROWMAJOR, (heads, 1, s_, s_),
                          "heads")
                self._node(op=P.OP_GEMM, in0=self.index[x], in1=self.index[x],
                           out=self.index[out], m=s_, n=s_, kk=dh, batch=heads, trans_b=1,
                           lda=three_h, ldb=three_h, ldc=s_, off_a=0, off_b=hid, off_c=0,
                           stride_a=dh, stride_b=dh, stride_c=s_ * s_, act=0, solution=sol)
            elif op == "pv":
                heads, dh = L["heads"], L["head_dim"]
                qkv = L["inputs"][1]
                s_, three_h = self.dims[qkv][2], self.dims[qkv][3]
                hid = three_h // 3
                self._new(out, (s_, hid), torch.bfloat16, P.ROWMAJOR, (1, 1, s_, hid), "matrix")
                self._node(op=P.OP_GEMM, in0=self.index[x], in1=self.index[qkv],
                           out=self.index[out], m=s_, n=dh, kk=s_, batch=heads, trans_b=0,
                           lda=s_, ldb=three_h, ldc=hid, off_a=0, off_b=2 * hid, off_c=0,
                           stride_a=s_ * s_, stride_b=dh, stride_c=dh, act=0, solution=sol)
            elif op == "attention":
                heads, dh = L["heads"], L["head_dim"]
                s_, three_h = self.dims[x][2], self.dims[x][3]
                hid = three_h // 3
                self._new(out, (s_, hid), torch.bfloat16, P.ROWMAJOR, (1, 1, s_, hid), "matrix")
                self._node(op=P.OP_ATTENTION, in0=self.index[x], out=self.index[out], m=s_,
                           n=heads, kk=dh, batch=1, scale=L["scale"], solution=sol)
            else:
                raise ValueError(op)
        self.inputs = [self.index[n] for n, _, _ in spec["inputs"]]
        self.outputs = [self.index[n] for n in spec["outputs"]]
        self._make_graph(None, 0)
        self.ws_bytes = P.workspace_bytes(self.graph)
        if self.alloc and self.ws_bytes:
            self.ws = torch.zeros(self.ws_bytes, dtype=torch.uint8, device=self.device)
            self._make_graph(self.ws.data_ptr(), self.ws_bytes)
        elif self.ws_bytes:  # host-only graph: a placeholder range like every tensor's
            self.ws = None
            self._make_graph(self._fake(self.ws_bytes), self.ws_bytes)
        else:
            self.ws = None

    def _make_graph(self, ws, ws_bytes):
        self._t_arr = (P.Tensor * len(self._tensors))(*self._tensors)
        self._n_arr = (P.Node * len(self._nodes))(*self._nodes)
        self._i_arr = (C.c_int32 * len(self.inputs))(*self.inputs)
        self._o_arr = (C.c_int32 * len(self.outputs))(*self.outputs)
        self.graph = P.Graph(len(self._tensors), self._t_arr, len(self._nodes), self._n_arr,
                             len(self.inputs), self._i_arr, len(self.outputs), self._o_arr,
                             ws, ws_bytes)

    # ------------------------------------------------------------ model image
    def save_image(self, path, x):
        """Write the lowered model as a model image for the native cold-start
        sampler (csrc/tools/pask_cold.cpp): header, the pask_tensor and
        pask_node arrays (device pointers replaced by blob ids, 1-based, 0 =
        none), the graph inputs / outputs, and the blobs -- every weight, bias,
        gamma, beta, and the input x in its device dtype.  Works for host-only
        graphs (alloc=False) too: no GPU is needed to write it."""
        import struct
        blobs, ids = [], {}

        def blob(ptr):
            if not ptr:
                return 0
            if ptr not in ids:
                ids[ptr] = len(blobs)
                h = self._blobs[ptr].contiguous()
                blobs.append(h.view(torch.uint8).numpy().tobytes())
            return ids[ptr] + 1

        nodes = (P.Node * len(self._nodes))()
        for i, nd in enumerate(self._nodes):
            C.memmove(C.byref(nodes[i]), C.byref(nd), C.sizeof(P.Node))
            for f in ("w", "bias", "gamma", "beta"):
                setattr(nodes[i], f, blob(getattr(nd, f)) or None)
        tensors = (P.Tensor * len(self._tensors))()
        for i, t in enumerate(self._tensors):
            C.memmove(C.byref(tensors[i]), C.byref(t), C.sizeof(P.Tensor))
            tensors[i].dptr = None
        (name, _, _), = self.spec["inputs"]
        dt = torch.float32 if self._tensors[self.index[name]].dtype == P.F32 else torch.bfloat16
        xin = torch.from_numpy(np.ascontiguousarray(x)).to(dt)
        input_blobs = [len(blobs)]
        blobs.append(xin.view(torch.uint8).numpy().tobytes())
        with open(path, "wb") as f:
            f.write(b"PASKMDL1")
            f.write(struct.pack("<6i", 1, len(self._tensors), len(self._nodes), len(self.inputs),
                                len(self.outputs), len(blobs)))
            f.write(struct.pack("<3Q", C.sizeof(P.Tensor), C.sizeof(P.Node), self.ws_bytes or 0))
            f.write(bytes(tensors))
            f.write(bytes(nodes))
            f.write(struct.pack(f"<{len(self.inputs)}i", *self.inputs))
            f.write(struct.pack(f"<{len(self.outputs)}i", *self.outputs))
            f.write(struct.pack(f"<{len(input_blobs)}i", *input_blobs))
            f.write(struct.pack(f"<{len(blobs)}Q", *[len(b) for b in blobs]))
            for b in blobs:
                f.write(b)
                f.write(b"\0" * ((-len(b)) % 256))
        return path

    def tensor_layout(self):
        """[(name, torch dtype, device shape, bytes)] in tensor order: how the
        native sampler's --dump file is laid out."""
        out = []
        names = sorted(self.index, key=self.index.get)
        for nm in names:
            t = self._tensors[self.index[nm]]
            nbytes = t.n * t.h * t.w * t.c * (4 if t.dtype == P.F32 else 2)
            out.append((nm, torch.float32 if t.dtype == P.F32 else torch.bfloat16, nbytes))
        return out

    # ------------------------------------------------------------ data movement
    def set_input(self, x):
        (name, _, dtype), = self.spec["inputs"]
        src = torch.from_numpy(np.ascontiguousarray(x))
        self.t[name].copy_(src.to(self.t[name].dtype))

    def read(self, name):
        """Device tensor -> float64 numpy in logical layout (NCHW images without
        channel padding, [rows, cols] matrices, [heads, S, S] scores)."""
        t = self.t[name].float().cpu().numpy().astype(np.float64)
        if self.kind[name] == "image" and t.ndim == 4 and self._tensors[self.index[name]].layout \
                != P.NCHW:
            lc = self.spec["tensors"][name][1]
            return t.transpose(0, 3, 1, 2)[:, :lc]
        return t

    def read_raw(self, name):
        return self.t[name].float().cpu().numpy().astype(np.float64)

    def write(self, name, arr_logical):
        """Write a logical-layout array into a device tensor (teacher forcing)."""
        t = self.t[name]
        a = np.asarray(arr_logical, dtype=np.float32)
        if self.kind[name] == "image" and t.ndim == 4 and self._tensors[self.index[name]].layout \
                != P.NCHW:
            full = np.zeros(tuple(t.shape), np.float32)
            full[..., :a.shape[1]] = a.transpose(0, 2, 3, 1)
            a = full
        t.copy_(torch.from_numpy(a.reshape(tuple(t.shape))).to(t.dtype))
