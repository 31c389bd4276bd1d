"""B200-native executor of stencil kernel DAGs with fission/fusion plans.

Thin ctypes binding of libstencilfuse.so (include/stencilfuse.h).  Argument
marshalling only: every step of the hot path (the generated sm_100a kernels,
the NCCL halo exchange) runs inside the library.  torch provides device
memory, streams and the process group; it computes nothing here.  If the
library is missing, import fails loudly — there is no fallback.

Method: Wahib & Maruyama, "Automated GPU Kernel Transformations in Large-Scale
Production Stencil Applications", HPDC'15.
"""
from __future__ import annotations

import ctypes
import os

from ._abi import (SP_F32, SP_F64, ROLE, SpArrayDesc, SpEdge, SpGrid, SpGroupReport, SpKernel,
                   SpLayout, SpSearchOptions, SpSearchReport, SpStmt, SpStmtRef, SpTerm, SpTap,
                   SpTileConfig, lib)

__all__ = ["Program", "Comm", "StencilError", "lib"]


class StencilError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"[sp_status {code}] {msg}")
        self.code = code


def _check(rc):
    if rc != 0:
        raise StencilError(rc, lib().sp_last_error().decode())


def _stream_handle(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    if hasattr(stream, "cuda_stream"):
        return ctypes.c_void_p(stream.cuda_stream)
    return ctypes.c_void_p(int(stream))


class Comm:
    """NCCL communicator for the z-slab decomposition, bootstrapped over torch.distributed."""

    def __init__(self, rank: int, world: int, group=None):
        import torch
        import torch.distributed as dist
        buf = (ctypes.c_ubyte * 128)()
        if rank == 0:
            _check(lib().sp_comm_unique_id(buf))
        t = torch.tensor(list(bytes(buf)), dtype=torch.uint8)
        if dist.is_initialized() and world > 1:
            backend = dist.get_backend(group)
            dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else "cpu"
            t = t.to(dev)
            dist.broadcast(t, src=0, group=group)
            t = t.cpu()
        raw = (ctypes.c_ubyte * 128)(*t.tolist())
        self.handle = ctypes.c_void_p()
        _check(lib().sp_comm_create(raw, world, rank, ctypes.byref(self.handle)))
        self.rank, self.world = rank, world

    @classmethod
    def loopback(cls, world: int):
        """Test transport: `world` in-process virtual ranks on the current device
        (sp_comm_create_loopback).  Drive each rank's Program from its own thread."""
        hs = (ctypes.c_void_p * world)()
        _check(lib().sp_comm_create_loopback(world, hs))
        out = []
        for r in range(world):
            c = cls.__new__(cls)
            c.handle = ctypes.c_void_p(hs[r])
            c.rank, c.world = r, world
            out.append(c)
        return out

    def __del__(self):
        h = getattr(self, "handle", None)
        if h:
            try:
                lib().sp_comm_destroy(h)
            except Exception:  # interpreter shutdown
                pass
            self.handle = None


def _parse_member(prog, ref):
    """'K' -> all statements of kernel K; 'K:i' -> statement i of K."""
    kidx = {k["name"]: i for i, k in enumerate(prog["kernels"])}
    if ":" in ref:
        k, s = ref.rsplit(":", 1)
        return [(kidx[k], int(s))]
    k = kidx[ref]
    return [(k, s) for s in range(len(prog["kernels"][k]["stmts"]))]


class Program:
    """A stencil program (kernels over shared 3-D arrays) bound to device memory.

    prog: dict in the synth/programs.py schema.  For a z-slab of a decomposed
    grid pass nz_global / z_offset / zhalo and a Comm.
    """

    def __init__(self, prog: dict, comm: Comm | None = None, nz_global=None, z_offset=0,
                 zhalo=0, options: dict | None = None):
        self.prog = prog
        self.dtype = prog["dtype"]
        g = prog["grid"]
        self.n = (int(g["nx"]), int(g["ny"]), int(g["nz"]))
        self.ghost = tuple(int(v) for v in g["ghost"])
        self.names = [a["name"] for a in prog["arrays"]]
        self.index = {a: i for i, a in enumerate(self.names)}
        grid = SpGrid(nx=self.n[0], ny=self.n[1], nz_local=self.n[2],
                      nz_global=int(nz_global or self.n[2]), z_offset=int(z_offset),
                      ghost=(ctypes.c_int32 * 3)(*self.ghost), zhalo=int(zhalo),
                      dtype=SP_F64 if self.dtype == "f64" else SP_F32)
        arrays = (SpArrayDesc * len(self.names))()
        self._keep = []
        for i, a in enumerate(prog["arrays"]):
            nm = a["name"].encode()
            self._keep.append(nm)
            arrays[i].name = nm
            arrays[i].role = ROLE[a["role"]]
        kernels = (SpKernel * len(prog["kernels"]))()
        for ki, k in enumerate(prog["kernels"]):
            stmts = (SpStmt * len(k["stmts"]))()
            for si, s in enumerate(k["stmts"]):
                terms = (SpTerm * len(s["terms"]))()
                for ti, t in enumerate(s["terms"]):
                    terms[ti].coef = float(t["c"])
                    terms[ti].a = self._tap(t["a"])
                    if "b" in t:
                        terms[ti].has_b = 1
                        terms[ti].b = self._tap(t["b"])
                stmts[si].out = self.index[s["out"]]
                stmts[si].n_terms = len(s["terms"])
                stmts[si].terms = terms
                self._keep.append(terms)
            nm = k["name"].encode()
            self._keep += [stmts, nm]
            kernels[ki].name = nm
            kernels[ki].n_stmts = len(k["stmts"])
            kernels[ki].stmts = stmts
            if k.get("box") is not None:
                box = (ctypes.c_int64 * 6)(*[int(v) for v in k["box"]])
                self._keep.append(box)
                kernels[ki].box = box
        self.comm = comm
        self.handle = ctypes.c_void_p()
        _check(lib().stencil_program_create(ctypes.byref(grid), len(self.names), arrays,
                                            len(prog["kernels"]), kernels,
                                            comm.handle if comm else None,
                                            ctypes.byref(self.handle)))
        lay = SpLayout()
        _check(lib().stencil_program_layout(self.handle, ctypes.byref(lay)))
        self.layout = {f: getattr(lay, f) for f, _ in SpLayout._fields_}
        self.tensors = {}
        for k, v in (options or {}).items():
            self.set_option(k, v)

    def _tap(self, t):
        return SpTap(self.index[t[0]], int(t[1]), int(t[2]), int(t[3]))

    def __del__(self):
        h = getattr(self, "handle", None)
        if h:
            try:
                lib().stencil_program_destroy(h)
            except Exception:  # interpreter shutdown
                pass
            self.handle = None

    # ---------------------------------------------------------- memory
    @property
    def elem(self):
        return 8 if self.dtype == "f64" else 4

    def alloc_shape(self):
        L = self.layout
        return (L["z_alloc"], L["y_alloc"], L["x_pitch"])

    def allocate(self, device, names=None, fill=float("nan")):
        """Allocate (torch) and bind every array; returns {name: tensor [z][y][x_pitch]}."""
        import torch
        dt = torch.float64 if self.dtype == "f64" else torch.float32
        for name in names or self.names:
            t = torch.full(self.alloc_shape(), fill, dtype=dt, device=device)
            self.bind(name, t)
        return self.tensors

    def bind(self, name, tensor):
        assert tensor.is_contiguous() and tensor.numel() * tensor.element_size() >= self.layout["bytes"]
        self.tensors[name] = tensor
        _check(lib().stencil_program_bind(self.handle, self.index[name],
                                          ctypes.c_void_p(tensor.data_ptr())))

    # ---------------------------------------------------------- peer push (option xpush)
    def temp_names(self):
        return [a["name"] for a in self.prog["arrays"] if a["role"] == "temp"]

    def signal_buffer(self):
        """Device address of this program's 64-B signal block (sp_signal_buffer)."""
        out = ctypes.c_void_p()
        _check(lib().sp_signal_buffer(self.handle, ctypes.byref(out)))
        return out.value

    def bind_peer(self, name, side, ptr):
        _check(lib().sp_bind_peer(self.handle, self.index[name], int(side), ctypes.c_void_p(ptr)))

    def bind_peer_signal(self, side, ptr):
        _check(lib().sp_bind_peer_signal(self.handle, int(side), ctypes.c_void_p(ptr)))

    @staticmethod
    def connect_peers_local(progs):
        """Peer-push wiring of in-process ranks (loopback virtual ranks on one device):
        each rank's neighbour buffers are the neighbours' own tensors."""
        for r, p in enumerate(progs):
            for side, q in ((0, r - 1), (1, r + 1)):
                if 0 <= q < len(progs):
                    for n in p.temp_names():
                        p.bind_peer(n, side, progs[q].tensors[n].data_ptr())
                    p.bind_peer_signal(side, progs[q].signal_buffer())

    def connect_peers(self, rank, world, group=None):
        """Peer-push wiring across processes: CUDA IPC handles of every TEMP array and
        of the signal block, all-gathered over torch.distributed, opened for the two
        z-neighbours (collective over the group)."""
        import torch.distributed as dist
        mine = {}
        for n in self.temp_names() + ["__signal__"]:
            ptr = self.signal_buffer() if n == "__signal__" else self.tensors[n].data_ptr()
            h = (ctypes.c_ubyte * 64)()
            off = ctypes.c_int64()
            _check(lib().sp_ipc_export(ctypes.c_void_p(ptr), h, ctypes.byref(off)))
            mine[n] = (bytes(h), off.value)
        allv = [None] * world
        dist.all_gather_object(allv, mine, group=group)
        for side, q in ((0, rank - 1), (1, rank + 1)):
            if not 0 <= q < world:
                continue
            for n, (h, off) in allv[q].items():
                out = ctypes.c_void_p()
                hb = (ctypes.c_ubyte * 64)(*h)
                _check(lib().sp_ipc_open(hb, off, ctypes.byref(out)))
                if n == "__signal__":
                    self.bind_peer_signal(side, out.value)
                else:
                    self.bind_peer(n, side, out.value)

    def padded_view(self, tensor, hz=None):
        """View of the dense padded region [nz+2hz][ny+2hy][nx+2hx] (ghost width per side)."""
        L = self.layout
        hx, hy, gz = self.ghost
        hz = gz if hz is None else hz
        nx, ny, nz = self.n
        return tensor[L["origin_z"] - hz:L["origin_z"] + nz + hz,
                      L["origin_y"] - hy:L["origin_y"] + ny + hy,
                      L["origin_x"] - hx:L["origin_x"] + nx + hx]

    def interior_view(self, tensor):
        L = self.layout
        nx, ny, nz = self.n
        return tensor[L["origin_z"]:L["origin_z"] + nz, L["origin_y"]:L["origin_y"] + ny,
                      L["origin_x"]:L["origin_x"] + nx]

    # ---------------------------------------------------------- program info
    def set_option(self, key, value):
        _check(lib().sp_program_set_option(self.handle, key.encode(), int(value)))

    def edges(self):
        n = ctypes.c_int32()
        _check(lib().sp_program_edges(self.handle, 0, None, ctypes.byref(n)))
        buf = (SpEdge * max(n.value, 1))()
        _check(lib().sp_program_edges(self.handle, n.value, buf, ctypes.byref(n)))
        return [(e.frm, e.to, e.kind, e.array) for e in buf[:n.value]]

    def fission(self, kernel):
        ki = kernel if isinstance(kernel, int) else [k["name"] for k in self.prog["kernels"]].index(kernel)
        ns = len(self.prog["kernels"][ki]["stmts"])
        comp = (ctypes.c_int32 * ns)()
        nc = ctypes.c_int32()
        _check(lib().sp_fission_components(self.handle, ki, comp, ctypes.byref(nc)))
        return list(comp), nc.value

    # ---------------------------------------------------------- plans
    def set_plan(self, groups):
        """groups: list of lists of member refs ('K' or 'K:i'), in execution order."""
        begin, members = [0], []
        for g in groups:
            for ref in g:
                members += _parse_member(self.prog, ref)
            begin.append(len(members))
        b = (ctypes.c_int32 * len(begin))(*begin)
        m = (SpStmtRef * len(members))(*[SpStmtRef(k, s) for k, s in members])
        _check(lib().fusion_plan_set(self.handle, len(groups), b, m))

    def plan_greedy(self):
        """Greedy fission/fusion plan from the library's model; list of groups of 'K:i' refs."""
        ng = ctypes.c_int32()
        _check(lib().sp_plan_greedy(self.handle, 0, ctypes.byref(ng), None, None))
        nst = sum(len(k["stmts"]) for k in self.prog["kernels"])
        begin = (ctypes.c_int32 * (ng.value + 1))()
        mem = (SpStmtRef * nst)()
        _check(lib().sp_plan_greedy(self.handle, ng.value, ctypes.byref(ng), begin, mem))
        names = [k["name"] for k in self.prog["kernels"]]
        return [[f"{names[mem[i].kernel]}:{mem[i].stmt}" for i in range(begin[g], begin[g + 1])]
                for g in range(ng.value)]

    def plan_search(self, generations=60, population=24, seed=1):
        """GGA-lite fission/fusion plan search over the library's model (sp_plan_search)."""
        ng = ctypes.c_int32()
        args = (self.handle, int(generations), int(population), ctypes.c_uint64(seed))
        _check(lib().sp_plan_search(*args, 0, ctypes.byref(ng), None, None))
        nst = sum(len(k["stmts"]) for k in self.prog["kernels"])
        begin = (ctypes.c_int32 * (ng.value + 1))()
        mem = (SpStmtRef * nst)()
        _check(lib().sp_plan_search(*args, ng.value, ctypes.byref(ng), begin, mem))
        names = [k["name"] for k in self.prog["kernels"]]
        return [[f"{names[mem[i].kernel]}:{mem[i].stmt}" for i in range(begin[g], begin[g + 1])]
                for g in range(ng.value)]

    def plan_search_ex(self, generations=30, population=24, seed=1, objective="model",
                       max_group_kernels=0, reps=0, c_violation=0.0, c_sm=0.0, configs=None,
                       stream=None, with_configs=False):
        """Lazy-fission plan search (sp_plan_search_ex): objective "model" (host) or
        "measured" (groups JIT-compiled and timed on the current device at the chooser's
        and each candidate configuration in `configs`; arrays must be bound).  Returns
        (plan, report dict) or, with_configs, (plan, per-group configuration dicts, report)."""
        def abi(c):  # option-level dict (as for tune) -> ABI values (zqueue/fastpath + 1)
            v = {k: int(x) for k, x in c.items() if k in dict(SpTileConfig._fields_)}
            for k in ("zqueue", "fastpath", "frame"):
                if k in v:
                    v[k] += 1
            return SpTileConfig(**v)
        cands = [abi(c) for c in (configs or [])]
        carr = (SpTileConfig * max(1, len(cands)))(*cands)
        o = SpSearchOptions(generations=int(generations), population=int(population),
                            seed=int(seed), objective={"model": 0, "measured": 1}[objective],
                            max_group_kernels=int(max_group_kernels), reps=int(reps),
                            c_violation=float(c_violation), c_sm=float(c_sm),
                            n_configs=len(cands), configs=carr)
        rep = SpSearchReport()
        ng = ctypes.c_int32()
        nst = sum(len(k["stmts"]) for k in self.prog["kernels"])
        begin = (ctypes.c_int32 * (nst + 1))()
        mem = (SpStmtRef * nst)()
        out_cfg = (SpTileConfig * nst)()
        sh = _stream_handle(stream) if objective == "measured" else None
        _check(lib().sp_plan_search_ex(self.handle, ctypes.byref(o), sh, nst, ctypes.byref(ng), begin, mem,
                                       out_cfg, ctypes.byref(rep)))
        names = [k["name"] for k in self.prog["kernels"]]
        plan = [[f"{names[mem[i].kernel]}:{mem[i].stmt}" for i in range(begin[g], begin[g + 1])]
                for g in range(ng.value)]
        report = {f: getattr(rep, f) for f, _ in SpSearchReport._fields_}
        if not with_configs:
            return plan, report
        cfgs = []
        for g in range(ng.value):
            c = {f: getattr(out_cfg[g], f) for f, _ in SpTileConfig._fields_ if getattr(out_cfg[g], f)}
            for k in ("zqueue", "fastpath", "frame"):  # back to option-level values (as tune() takes)
                if k in c:
                    c[k] -= 1
            cfgs.append(c or None)
        return plan, cfgs, report

    def n_launches(self, mode):
        n = ctypes.c_int32()
        _check(lib().sp_plan_count(self.handle, self._mode(mode), ctypes.byref(n)))
        return n.value

    def report(self, mode, i):
        r = SpGroupReport()
        _check(lib().sp_plan_report(self.handle, self._mode(mode), i, ctypes.byref(r)))
        d = {f: getattr(r, f) for f, _ in SpGroupReport._fields_}
        d["ext"] = list(r.ext)
        return d

    def reports(self, mode):
        return [self.report(mode, i) for i in range(self.n_launches(mode))]

    def source(self, mode):
        n = ctypes.c_size_t()
        _check(lib().sp_plan_source(self.handle, self._mode(mode), None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value + 1)
        _check(lib().sp_plan_source(self.handle, self._mode(mode), buf, n.value + 1, ctypes.byref(n)))
        return buf.value.decode()

    def tune(self, mode, i, cfg):
        """Pin launch i's configuration: dict with tile_x, tile_y, zchunk, threads, prefetch,
        block_x, block_y, block_cby (missing/0 = chooser), zqueue (the option's values
        0/1/2), fastpath and frame (0/1; missing = the program option); None removes the pin."""
        if cfg is None:
            _check(lib().sp_plan_tune(self.handle, self._mode(mode), i, None))
            return
        vals = {k: int(v) for k, v in cfg.items() if k in dict(SpTileConfig._fields_)}
        for k in ("zqueue", "fastpath", "frame"):
            if k in vals:
                vals[k] += 1  # ABI: 0 = inherit the program option, value + 1 otherwise
        c = SpTileConfig(**vals)
        _check(lib().sp_plan_tune(self.handle, self._mode(mode), i, ctypes.byref(c)))

    def exchange_plan(self, mode, i):
        """[(array name, planes below, planes above)] the executor receives into the
        ghost planes right before launch i on several ranks (sp_plan_exchange)."""
        n = ctypes.c_int32()
        k = len(self.names)
        buf, lo, hi = (ctypes.c_int32 * k)(), (ctypes.c_int32 * k)(), (ctypes.c_int32 * k)()
        _check(lib().sp_plan_exchange(self.handle, self._mode(mode), i, k, buf, lo, hi,
                                      ctypes.byref(n)))
        return [(self.names[buf[j]], lo[j], hi[j]) for j in range(n.value)]

    def wave_offsets(self):
        """Plane skew of each fused launch in the z-wave schedule (option "zwave")."""
        n = ctypes.c_int32()
        _check(lib().sp_plan_wave_offsets(self.handle, 0, None, ctypes.byref(n)))
        buf = (ctypes.c_int32 * max(1, n.value))()
        _check(lib().sp_plan_wave_offsets(self.handle, n.value, buf, ctypes.byref(n)))
        return [buf[j] for j in range(n.value)]

    def load(self, mode):
        """Compile if needed and load the mode's kernels on the current device (sp_load)."""
        _check(lib().sp_load(self.handle, self._mode(mode)))

    def compile(self, mode):
        _check(lib().sp_compile(self.handle, self._mode(mode)))

    @staticmethod
    def _mode(mode):
        return {"unfused": 0, "fused": 1, 0: 0, 1: 1}[mode]

    # ---------------------------------------------------------- execution
    def run_unfused(self, stream=None):
        _check(lib().run_unfused(self.handle, _stream_handle(stream)))

    def run_fused(self, stream=None):
        _check(lib().run_fused(self.handle, _stream_handle(stream)))

    def run(self, mode, stream=None):
        (self.run_fused if self._mode(mode) else self.run_unfused)(stream)

    def dag(self, mode="fused"):
        """[(dependencies, stream index)] per launch (sp_plan_dag): the launch DAG run_fused
        follows with the options "rename" / "streams"."""
        out = []
        for i in range(self.n_launches(mode)):
            buf = (ctypes.c_int32 * 64)()
            nd, st = ctypes.c_int32(), ctypes.c_int32()
            _check(lib().sp_plan_dag(self.handle, self._mode(mode), i, 64, buf, ctypes.byref(nd),
                                     ctypes.byref(st)))
            out.append((list(buf[:min(nd.value, 64)]), st.value))
        return out

    def run_launch(self, mode, i, stream=None):
        _check(lib().sp_run_launch(self.handle, self._mode(mode), i, _stream_handle(stream)))

    def launch_count(self, mode):
        """Kernel launches one run_unfused / run_fused call issues (sp_run_launch_count)."""
        n = ctypes.c_int32()
        _check(lib().sp_run_launch_count(self.handle, self._mode(mode), ctypes.byref(n)))
        return n.value

    def exchange_halos(self, names, depth, stream=None):
        arr = (ctypes.c_int32 * len(names))(*[self.index[n] for n in names])
        _check(lib().exchange_halos(self.handle, len(names), arr, depth, _stream_handle(stream)))
