"""paper_conf_ispass_maxw23_b200 -- B200-native batched TFHE gate bootstrapping (PyTFHE's hot path).

Thin Python binding over the C ABI of libtfhe_b200.so (include/tfhe_b200.h); same names, argument
marshalling only.  PyTorch provides device memory (ciphertexts live in int32 CUDA tensors whose bits are the
u32 torus words), streams and process groups; every step of a gate runs in the sm_100a kernels.

    ctx = Context()                      # cuda:0, tfhe-lib 128-bit parameters
    ctx.load_keys(bk, ksk)               # host u32 arrays from the client's KeyGen
    out = ctx.gates(NAND, ca, cb)        # batched bootstrapped gates
    dnet = ctx.upload(netlist)           # Algorithm-1 levelisation + descriptors
    ctx.run_netlist(dnet, wires)         # level by level on one GPU, or sharded over a process group

P:N = /root/reference/PAPER.md line N.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _native, parallel
from ._native import TBError, build
from .netlist import (AND, ANDNY, ANDYN, BINARY_GATES, GATE_CODES, MUX, NAND, NOR, NOT, OR, ORNY, ORYN, XNOR, XOR,
                      Netlist, read_pytfhe_binary, write_pytfhe_binary)

N_LWE = 630            # n
N_RING = 1024          # N
CT_WORDS = N_LWE + 1   # 631 words per LWE ciphertext (2524 B = the paper's 2.46 KB)
EXT_WORDS = N_RING + 1
WIRE_STRIDE = 632      # default row stride of wire arrays (16-byte aligned rows)
BK_WORDS = N_LWE * 6 * 2 * N_RING
KSK_WORDS = N_RING * 8 * 4 * CT_WORDS

__all__ = ["Context", "DevNetlist", "Netlist", "TBError", "build", "read_pytfhe_binary", "write_pytfhe_binary",
           "GATE_CODES", "NAND", "AND", "OR", "NOR", "XOR", "XNOR", "ANDNY", "ANDYN", "ORNY", "ORYN", "NOT", "MUX",
           "CT_WORDS", "WIRE_STRIDE", "BK_WORDS", "KSK_WORDS", "version"]


def version() -> str:
    return _native.lib().tb_version().decode()


def _nullcontext():
    import contextlib
    return contextlib.nullcontext()


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream_handle(stream=None):
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _check_dev(t: torch.Tensor, device: torch.device, name: str):
    if t.device != device or t.dtype != torch.int32 or t.dim() != 2 or t.stride(1) != 1:
        raise ValueError("%s must be a 2-D int32 tensor on %s with unit inner stride" % (name, device))


class DevNetlist:
    """Library-owned device copy of a levelised netlist (tb_netlist_upload)."""

    def __init__(self, ctx: "Context", net: Netlist):
        self.ctx, self.net = ctx, net
        h = ctypes.c_void_p()
        s = net.c_struct()
        _native.check(_native.lib().tb_netlist_upload(ctx._h, ctypes.byref(s), ctypes.byref(h)))
        self._h = h
        nl, nr = ctypes.c_int64(), ctypes.c_int64()
        _native.check(_native.lib().tb_netlist_info(h, ctypes.byref(nl), ctypes.byref(nr)))
        self.n_levels, self.n_rows = int(nl.value), int(nr.value)
        self.row_of_wire = np.zeros(net.n_wires, np.int64)
        _native.check(_native.lib().tb_netlist_wire_rows(h, self.row_of_wire.ctypes.data))
        self.levels = []          # (row0, n_gates, n_boot, n_lanes) per level 1..n_levels
        for L in range(1, self.n_levels + 1):
            v = [ctypes.c_int64() for _ in range(4)]
            _native.check(_native.lib().tb_netlist_level(h, L, *[ctypes.byref(x) for x in v]))
            self.levels.append(tuple(int(x.value) for x in v))
        w = ctypes.c_int()
        _native.check(_native.lib().tb_netlist_world(h, ctypes.byref(w)))
        self.world = int(w.value)     # ranks the level order was planned for (tb_set_plan_world)

    def early(self, rank: int):
        """per level, this rank's early-gate count (tb_netlist_early); needs world == the loop's world size"""
        out = []
        for L in range(1, self.n_levels + 1):
            e = ctypes.c_int64()
            _native.check(_native.lib().tb_netlist_early(self._h, L, rank, ctypes.byref(e)))
            out.append(int(e.value))
        return out

    @property
    def n_boot(self) -> int:
        return sum(lv[2] for lv in self.levels)

    def free(self):
        if self._h:
            _native.lib().tb_netlist_free(self.ctx._h, self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Context:
    """One device, keys resident in HBM (BK in the NTT domain 92.9 MB, KSK 62.1 MB)."""

    def __init__(self, device=0):
        self.device = torch.device("cuda", device if isinstance(device, int) else torch.device(device).index or 0)
        L = _native.lib()
        p = L.tb_default_params()
        h = ctypes.c_void_p()
        _native.check(L.tb_ctx_create(ctypes.byref(p), self.device.index, ctypes.byref(h)))
        self._h = h

    # ---- keys (the public key is broadcast to the workers before traversal) ----
    def load_bk(self, bk: np.ndarray):
        bk = np.ascontiguousarray(bk, np.uint32).reshape(-1)
        _native.check(_native.lib().tb_load_bk(self._h, bk.ctypes.data, bk.size))

    def load_ksk(self, ksk: np.ndarray):
        ksk = np.ascontiguousarray(ksk, np.uint32).reshape(-1)
        _native.check(_native.lib().tb_load_ksk(self._h, ksk.ctypes.data, ksk.size))

    def load_keys(self, bk: np.ndarray, ksk: np.ndarray):
        self.load_bk(bk)
        self.load_ksk(ksk)

    def set_lanes_per_cta(self, lanes: int):
        """1..4 fixed, 0 = auto per launch (the default)."""
        _native.check(_native.lib().tb_set_lanes_per_cta(self._h, lanes))

    def br6_lanes_per_cta(self, nlanes: int) -> int:
        """Lanes per CTA the default blind-rotation kernel uses for a launch of `nlanes` lanes."""
        rc = _native.lib().tb_br6_lanes_per_cta(self._h, nlanes)
        if rc < 0:
            _native.check(rc)
        return rc

    def set_br_variant(self, variant: int):
        """6 = br6_kernel (default), 10 = brf_kernel (FP64 pipe), 12 = brt_kernel (tensor cores), 14 = br6t_kernel
        (br6 with its forward NTT on the tensor cores); bit-identical."""
        _native.check(_native.lib().tb_set_br_variant(self._h, variant))

    def set_narrow_lanes(self, lanes: int):
        """levels with <= lanes bootstraps run in latency mode (see set_narrow_kernel); 0 disables"""
        _native.check(_native.lib().tb_set_narrow_lanes(self._h, lanes))

    def set_level_capacity(self, lanes: int):
        """netlist uploads: keep levels within `lanes` bootstraps where slack allows (-1 auto, 0 = Algorithm 1)"""
        _native.check(_native.lib().tb_set_level_capacity(self._h, lanes))

    def set_narrow_kernel(self, kernel: int):
        """latency-mode kernel: 0 = auto (default), 11 = brl (4-SM cluster), 9 = br9 (2-SM cluster), 13 = brtl (1 SM, tensor cores)"""
        _native.check(_native.lib().tb_set_narrow_kernel(self._h, kernel))

    def set_ks_tile(self, gates: int):
        """gates per key-switch CTA: 8 (default), 16 or 32"""
        _native.check(_native.lib().tb_set_ks_tile(self._h, gates))

    # ---- tensors ----
    def empty(self, rows: int, stride: int = WIRE_STRIDE) -> torch.Tensor:
        return torch.empty((rows, stride), dtype=torch.int32, device=self.device)

    def to_device(self, cts: np.ndarray, stride: int = WIRE_STRIDE) -> torch.Tensor:
        cts = np.asarray(cts, np.uint32)
        t = torch.zeros((cts.shape[0], stride), dtype=torch.int32)
        t[:, :cts.shape[1]] = torch.from_numpy(cts.view(np.int32))
        return t.to(self.device)

    @staticmethod
    def to_host(t: torch.Tensor, words: int = CT_WORDS) -> np.ndarray:
        return t[:, :words].cpu().numpy().view(np.uint32).copy()

    # ---- batched gates (P:54 bootstrapped-Gate) ----
    def gates(self, gate: int, ca: torch.Tensor, cb: torch.Tensor = None, cc: torch.Tensor = None,
              out: torch.Tensor = None, stream=None) -> torch.Tensor:
        _check_dev(ca, self.device, "ca")
        for name, t in (("cb", cb), ("cc", cc)):
            if t is not None:
                _check_dev(t, self.device, name)
                if t.shape != ca.shape or t.stride() != ca.stride():
                    raise ValueError("%s must match ca's shape and stride" % name)
        out = torch.empty_like(ca) if out is None else out
        _check_dev(out, self.device, "out")
        _native.check(_native.lib().tb_gates(self._h, gate, _ptr(ca), _ptr(cb), _ptr(cc), _ptr(out), ca.shape[0],
                                             ca.stride(0), _stream_handle(stream)))
        return out

    def gates_host(self, gate: int, ca: np.ndarray, cb: np.ndarray = None, cc: np.ndarray = None) -> np.ndarray:
        """End-to-end through host buffers (H2D, gates, D2H inside the call)."""
        ca = np.ascontiguousarray(ca, np.uint32)
        cb = None if cb is None else np.ascontiguousarray(cb, np.uint32)
        cc = None if cc is None else np.ascontiguousarray(cc, np.uint32)
        out = np.empty_like(ca)
        vp = lambda a: None if a is None else a.ctypes.data
        _native.check(_native.lib().tb_gates_host(self._h, gate, vp(ca), vp(cb), vp(cc), out.ctypes.data,
                                                  ca.shape[0], ca.shape[1]))
        return out

    def bootstrap_wo_ks(self, cts: torch.Tensor, out: torch.Tensor = None, stream=None) -> torch.Tensor:
        _check_dev(cts, self.device, "cts")
        out = torch.empty((cts.shape[0], 1028), dtype=torch.int32, device=self.device) if out is None else out
        _native.check(_native.lib().tb_bootstrap_wo_ks(self._h, _ptr(cts), cts.stride(0), _ptr(out), out.stride(0),
                                                       cts.shape[0], _stream_handle(stream)))
        return out

    def keyswitch(self, ext: torch.Tensor, out: torch.Tensor = None, stream=None) -> torch.Tensor:
        _check_dev(ext, self.device, "ext")
        out = self.empty(ext.shape[0]) if out is None else out
        _native.check(_native.lib().tb_keyswitch(self._h, _ptr(ext), ext.stride(0), _ptr(out), out.stride(0),
                                                 ext.shape[0], _stream_handle(stream)))
        return out

    def ntt_muladd6(self, digits: torch.Tensor, polys: torch.Tensor) -> torch.Tensor:
        res = torch.empty(N_RING, dtype=torch.int32, device=self.device)
        _native.check(_native.lib().tb_ntt_muladd6(self._h, _ptr(digits.contiguous()), _ptr(polys.contiguous()),
                                                   _ptr(res)))
        return res

    def fft_muladd6(self, digits: torch.Tensor, polys: torch.Tensor) -> torch.Tensor:
        res = torch.empty(N_RING, dtype=torch.int32, device=self.device)
        _native.check(_native.lib().tb_fft_muladd6(self._h, _ptr(digits.contiguous()), _ptr(polys.contiguous()),
                                                   _ptr(res)))
        return res

    def microbench(self, iters: int = 4096):
        b, m = ctypes.c_double(), ctypes.c_double()
        _native.check(_native.lib().tb_microbench(self._h, iters, ctypes.byref(b), ctypes.byref(m)))
        return b.value, m.value

    def microbench_fields(self, iters: int = 4096) -> dict:
        """measured butterfly / MAC rates of the 30-bit field and of Goldilocks (tb_microbench_fields)"""
        r = (ctypes.c_double * 4)()
        _native.check(_native.lib().tb_microbench_fields(self._h, iters, r))
        return {"shoup30_bfly_per_s": r[0], "goldilocks_bfly_per_s": r[1], "goldilocks_shift_bfly_per_s": r[2],
                "mac64_per_s": r[3]}

    def tc_muladd(self, digits: torch.Tensor, polys: torch.Tensor) -> torch.Tensor:
        """diagnostic: [4][2][1024] = sum_r digits[g][r] (x) polys[r][q] through the tensor-core CMux (tb_tc_muladd)"""
        res = torch.empty((4, 2, N_RING), dtype=torch.int32, device=self.device)
        d, p = digits.contiguous(), polys.contiguous()
        _native.check(_native.lib().tb_tc_muladd(self._h, _ptr(d), _ptr(p), _ptr(res)))
        return res

    def tc_mma_test(self, A: np.ndarray, B: np.ndarray, a_signed: bool = False, b_signed: bool = False,
                    lbo: int = 128) -> np.ndarray:
        """diagnostic: A [128][K] . B [N][K]^T as s32 through tcgen05.mma kind::i8 (tb_tc_mma_test)"""
        a = torch.from_numpy(np.ascontiguousarray(A).view(np.uint8)).to(self.device)
        b = torch.from_numpy(np.ascontiguousarray(B).view(np.uint8)).to(self.device)
        d = torch.empty((128, B.shape[0]), dtype=torch.int32, device=self.device)
        _native.check(_native.lib().tb_tc_mma_test(self._h, _ptr(a), _ptr(b), A.shape[1], B.shape[0], int(a_signed),
                                                   int(b_signed), lbo, _ptr(d)))
        return d.cpu().numpy()

    def key_bytes(self) -> int:
        v = ctypes.c_size_t()
        _native.check(_native.lib().tb_key_bytes(self._h, ctypes.byref(v)))
        return int(v.value)

    # ---- netlists (Algorithm 1) ----
    def upload(self, net: Netlist, world: int = 1) -> DevNetlist:
        """Levelise and upload; world > 1 orders every level for a loop over that many ranks so each rank's chunk
        starts with the gates it can run before the previous level's exchange (tb_set_plan_world)."""
        _native.check(_native.lib().tb_set_plan_world(self._h, world))
        try:
            return DevNetlist(self, net)
        finally:
            _native.lib().tb_set_plan_world(self._h, 1)

    def wire_array(self, dnet: DevNetlist, slack_rows: int = 0, stride: int = WIRE_STRIDE) -> torch.Tensor:
        return torch.zeros((dnet.n_rows + slack_rows, stride), dtype=torch.int32, device=self.device)

    def run_level(self, dnet: DevNetlist, level: int, g0: int, g1: int, wires: torch.Tensor, stream=None):
        _check_dev(wires, self.device, "wires")
        _native.check(_native.lib().tb_run_level(self._h, dnet._h, level, g0, g1, _ptr(wires), wires.stride(0),
                                                 _stream_handle(stream)))

    def run_netlist(self, dnet: DevNetlist, wires: torch.Tensor, group=None, stream=None, exchange: str = "fused",
                    early_start: bool = True):
        """Evaluate every level.  Without a process group: one device (tb_run_netlist).  With one: each
        level's gates are split into R contiguous chunks and rank r evaluates chunk r; the level's output rows
        reach every rank either through the key-switch kernels' own stores into the peers' wire arrays
        (exchange="fused": CUDA-IPC peer memory, tb_set_peer_wires, then a barrier) or through an in-place
        all-gather over the process group (exchange="allgather").  If dnet was uploaded for this world size
        (upload(net, world=R)) and the exchange is fused, each rank starts the next level's locally ready gates
        before the current level's barrier (early_start).  DESIGN.md "Multi-GPU"."""
        _check_dev(wires, self.device, "wires")
        if group is None:
            _native.check(_native.lib().tb_run_netlist(self._h, dnet._h, _ptr(wires), wires.stride(0),
                                                       _stream_handle(stream)))
            return
        if exchange not in ("fused", "allgather"):
            raise ValueError("exchange must be 'fused' or 'allgather'")
        levels = [(row0, ng) for row0, ng, _, _ in dnet.levels]
        run = lambda L, g0, g1: self.run_level(dnet, L, g0, g1, wires, stream)   # noqa: E731
        if exchange == "fused":
            self.attach_peers(wires, group)
        # the per-level barrier / all-gather must be ordered on the stream the level kernels run on: make it the
        # current stream for the loop (collectives order against torch's current stream)
        import torch.distributed as dist
        R, r = dist.get_world_size(group), dist.get_rank(group)
        early = dnet.early(r) if (dnet.world == R and R > 1 and early_start) else None
        with torch.cuda.stream(stream) if stream is not None else _nullcontext():
            parallel.level_loop(levels, wires, run, group, fused=exchange == "fused", early=early)

    # ---- fused all-gather: the other ranks' wire arrays mapped into this process (CUDA IPC) ----
    def attach_peers(self, wires: torch.Tensor, group):
        """Map every other rank's `wires` (same shape and stride) into this process and make tb_run_level's
        key-switch kernels store each output row into all of them (tb_set_peer_wires).  Collective over
        `group`; a no-op when this exact tensor is already attached."""
        import torch.distributed as dist
        key = (wires.data_ptr(), tuple(wires.shape), wires.stride(0))
        if getattr(self, "_peer_key", None) == key:
            return
        self.detach_peers()
        R, r = dist.get_world_size(group), dist.get_rank(group)
        h = (ctypes.c_ubyte * 64)()
        off = ctypes.c_int64()
        mine, err = None, None
        try:
            _native.check(_native.lib().tb_ipc_export(_ptr(wires), h, ctypes.byref(off)))
            mine = (bytes(h), off.value, tuple(wires.shape), wires.stride(0))
        except TBError as e:
            err = str(e)
        allh = [None] * R
        dist.all_gather_object(allh, mine, group=group)     # collective: every rank takes part, even on failure
        ptrs, bases = [], []
        err = None if mine is not None else err
        if err is None and any(x is None for x in allh):
            err = "a peer rank could not export its wire array"
        if err is None:
            try:
                for k, (hb, o, shape, stride) in enumerate(allh):
                    if k == r:
                        continue
                    if shape != tuple(wires.shape) or stride != wires.stride(0):
                        raise ValueError("rank %d's wire array has shape %s / stride %d, not %s / %d"
                                         % (k, shape, stride, tuple(wires.shape), wires.stride(0)))
                    p, b = ctypes.c_void_p(), ctypes.c_void_p()
                    buf = (ctypes.c_ubyte * 64).from_buffer_copy(hb)
                    _native.check(_native.lib().tb_ipc_import(self._h, buf, o, ctypes.byref(p), ctypes.byref(b)))
                    ptrs.append(p.value)
                    bases.append(b.value)
                arr = (ctypes.c_void_p * max(len(ptrs), 1))(*ptrs)
                _native.check(_native.lib().tb_set_peer_wires(self._h, _ptr(wires), arr, len(ptrs)))
            except (TBError, ValueError) as e:
                err = str(e)
        oks = [None] * R
        dist.all_gather_object(oks, err is None, group=group)   # all ranks attach, or none does
        if not all(oks):
            _native.lib().tb_set_peer_wires(self._h, None, None, 0)
            for b in bases:
                _native.lib().tb_ipc_close(self._h, ctypes.c_void_p(b))
            raise TBError(_native.TB_ECUDA,
                          "fused exchange unavailable: %s" % (err or "failed on another rank"))
        self._peer_bases, self._peer_key = bases, key

    def detach_peers(self):
        """Stop storing into peer arrays and unmap them."""
        bases = getattr(self, "_peer_bases", [])
        if getattr(self, "_h", None):
            _native.check(_native.lib().tb_set_peer_wires(self._h, None, None, 0))
            for b in bases:
                _native.lib().tb_ipc_close(self._h, ctypes.c_void_p(b))
        self._peer_bases, self._peer_key = [], None

    def set_host_overlap(self, enable: bool):
        """run_netlist_host*: overlap the host copies with the level loop (default) or serialise them"""
        _native.check(_native.lib().tb_set_host_overlap(self._h, 1 if enable else 0))

    def run_netlist_host(self, dnet: DevNetlist, inputs: np.ndarray, output_wires) -> np.ndarray:
        """End-to-end through HOST buffers (tb_run_netlist_host): input ciphertexts [n_inputs, >=631] u32 ->
        output ciphertexts [len(output_wires), 631] u32.  Pinned host memory makes the copies faster."""
        inputs = np.ascontiguousarray(inputs, np.uint32) if not isinstance(inputs, np.ndarray) or \
            inputs.dtype != np.uint32 or not inputs.flags.c_contiguous else inputs
        ow = np.ascontiguousarray(output_wires, np.int64)
        out = np.empty((ow.size, CT_WORDS), np.uint32)
        _native.check(_native.lib().tb_run_netlist_host(self._h, dnet._h, inputs.ctypes.data, inputs.shape[1],
                                                        ow.ctypes.data, ow.size, out.ctypes.data, CT_WORDS))
        return out

    def run_netlist_host_into(self, dnet: DevNetlist, inputs: torch.Tensor, output_wires: np.ndarray,
                              out: torch.Tensor) -> None:
        """Same with caller-owned (pinned) host tensors: inputs [n_inputs, stride] int32, out [n, stride]."""
        _native.check(_native.lib().tb_run_netlist_host(self._h, dnet._h, ctypes.c_void_p(inputs.data_ptr()),
                                                        inputs.stride(0), output_wires.ctypes.data,
                                                        output_wires.size, ctypes.c_void_p(out.data_ptr()),
                                                        out.stride(0)))

    # ---- end to end over a process group (sharded level loop with host buffers) ----
    def shard_io(self, dnet: DevNetlist, world: int, rank: int, output_wires=None):
        """I/O plan of rank `rank` of the sharded level loop (parallel.shard per level): the input rows its gate
        ranges read, and the (position in output_wires, wire row) pairs its gate ranges produce.  Host logic."""
        key = (world, rank, None if output_wires is None else np.asarray(output_wires, np.int64).tobytes())
        cache = dnet.__dict__.setdefault("_shard_io", {})
        if key in cache:
            return cache[key]
        net, ni = dnet.net, dnet.net.n_inputs
        order = np.argsort(dnet.row_of_wire[ni:], kind="stable")     # level-sorted position -> gate index
        mine = []
        for row0, ng, _, _ in dnet.levels:
            g0, g1, _ = parallel.shard(ng, world, rank)
            if g1 > g0:
                mine.append(np.arange(row0 - ni + g0, row0 - ni + g1))
        pos = np.concatenate(mine) if mine else np.zeros(0, np.int64)
        g = order[pos]
        ins = np.concatenate([net.in0[g], np.where(net.type[g] == NOT, -1, net.in1[g]),
                              np.where(net.type[g] == MUX, net.in2[g], -1)])
        ins = ins[(ins >= 0) & (ins < ni)]
        outs = []
        if output_wires is not None:
            ow = np.asarray(output_wires, np.int64)
            rows = dnet.row_of_wire[ow]
            produced = np.zeros(dnet.n_rows, bool)
            produced[ni + pos] = True
            if rank == 0:                    # outputs that are primary inputs (passed through): rank 0 returns them
                produced[:ni] = True
            k = np.nonzero(produced[rows])[0]
            outs = list(zip(k.tolist(), rows[k].tolist()))
            if rank == 0:
                ins = np.concatenate([ins, rows[rows < ni]])
        in_rows = np.unique(ins)
        cache[key] = (in_rows, outs)
        return cache[key]

    @staticmethod
    def _runs(a, b=None):
        """maximal runs where a (and b) advance by one together: [(a0, b0, length)]"""
        a = np.asarray(a, np.int64)
        b = a if b is None else np.asarray(b, np.int64)
        if a.size == 0:
            return []
        brk = np.nonzero((np.diff(a) != 1) | (np.diff(b) != 1))[0] + 1
        starts = np.concatenate([[0], brk])
        ends = np.concatenate([brk, [a.size]])
        return [(int(a[s]), int(b[s]), int(e - s)) for s, e in zip(starts, ends)]

    def run_netlist_host_sharded(self, dnet: DevNetlist, inputs: torch.Tensor, output_wires, out: torch.Tensor,
                                 wires: torch.Tensor, group, exchange: str = "fused", stream=None,
                                 inputs_row0: int = 0, out_pos0: int = 0):
        """End to end over a process group: this rank copies the input rows its gates read from host `inputs`
        (pinned int32 rows; inputs[k] = input row inputs_row0 + k) into `wires`, runs the sharded level loop
        (run_netlist with the group), copies the output rows its own gate ranges produced into `out` (pinned
        int32 rows; out[k] = output_wires[out_pos0 + k]) and synchronises.  Together the ranks return every
        output exactly once.  Returns (h2d_bytes, d2h_bytes) of this rank."""
        in_rows, outs = self.shard_io(dnet, dist_world(group), dist_rank(group), output_wires)
        if in_rows.size and (in_rows[0] < inputs_row0 or in_rows[-1] >= inputs_row0 + inputs.shape[0]):
            raise ValueError("host inputs do not cover the input rows this rank reads")
        if outs and (outs[0][0] < out_pos0 or outs[-1][0] >= out_pos0 + out.shape[0]):
            raise ValueError("host output buffer does not cover the outputs this rank produces")
        st = torch.cuda.current_stream(self.device) if stream is None else stream
        w = inputs.shape[1]
        with torch.cuda.stream(st):
            for a, _, n in self._runs(in_rows):
                wires[a:a + n, :w].copy_(inputs[a - inputs_row0:a - inputs_row0 + n], non_blocking=True)
        self.run_netlist(dnet, wires, group, stream=st, exchange=exchange)
        with torch.cuda.stream(st):
            for k, r, n in self._runs([k for k, _ in outs], [r for _, r in outs]):
                out[k - out_pos0:k - out_pos0 + n].copy_(wires[r:r + n, :out.shape[1]], non_blocking=True)
        st.synchronize()
        return int(in_rows.size) * w * 4, len(outs) * out.shape[1] * 4

    # ---- per-kernel device time (CUDA events around each launch) ----
    def profile(self, enable: bool):
        _native.check(_native.lib().tb_profile_enable(self._h, 1 if enable else 0))

    def profile_read(self):
        """-> (br_ms, br_launches, ks_ms, ks_launches) since profile(True)."""
        a, b, c, d = ctypes.c_double(), ctypes.c_int64(), ctypes.c_double(), ctypes.c_int64()
        _native.check(_native.lib().tb_profile_read(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c),
                                                    ctypes.byref(d)))
        return a.value, int(b.value), c.value, int(d.value)

    def close(self):
        if getattr(self, "_h", None):
            try:
                self.detach_peers()
            except Exception:
                pass
            _native.lib().tb_ctx_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def dist_world(group) -> int:
    import torch.distributed as dist
    return dist.get_world_size(group) if group is not None else 1


def dist_rank(group) -> int:
    import torch.distributed as dist
    return dist.get_rank(group) if group is not None else 0


def slack_rows(dnet: DevNetlist, world: int) -> int:
    """Extra wire rows needed so every level's padded all-gather stays inside the array."""
    return parallel.slack_rows([(row0, ng) for row0, ng, _, _ in dnet.levels], dnet.n_rows, world)
