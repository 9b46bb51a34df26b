"""B200-native GPApriori support counting (Zhang, Zhang & Bakos, IEEE Cluster 2011).

Thin Python binding over the C ABI of ``libgpapriori.so`` (``include/gpapriori.h``): argument
marshalling only -- every step of the path (validation, generation-1 histogram, static-bitset
build, support counting, NCCL all-reduce) runs in the library's sm_100a kernels and C++
runtime.  There is no CPU fallback: importing works without a GPU (so the ABI can be
inspected), but every compute call fails loudly if the library is missing or no B200 is
present.

    import paper_conf_cluster_zhangzb11a_b200 as gpa
    res = gpa.mine(offsets, items, n_items, min_count=gpa.min_count(n_tx, "0.01"))
    res.frequent(3)        # (n, 3) item ids and their supports

Inputs are CSR transaction lists: ``offsets`` (uint64/int64, n_tx+1) and ``items`` (uint32/int32).
numpy arrays / CPU tensors are host inputs (copied to the device inside the call, as the
paper copies its database to graphics memory, P18@755); CUDA tensors are device inputs used
in place.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from fractions import Fraction

import numpy as np

__all__ = [
    "GpaError", "lib", "version", "min_count", "Options", "Dist", "Bitset", "mine", "MineResult", "Rules",
    "KERNEL_AUTO", "KERNEL_V0", "KERNEL_PREFIX", "KERNEL_PAIRS", "KERNEL_TRIE", "KERNEL_PAIRS_TC", "KERNEL_PROJ",
    "KERNEL_FUSED", "PHASES",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libgpapriori.so")

KERNEL_AUTO, KERNEL_V0, KERNEL_PREFIX, KERNEL_PAIRS, KERNEL_TRIE, KERNEL_PAIRS_TC, KERNEL_PROJ, KERNEL_FUSED = range(8)
KERNEL_NAMES = {0: "auto", 1: "v0", 2: "prefix", 3: "pairs", 4: "trie", 5: "pairs_tc", 6: "proj", 7: "fused"}
KEEP_CANDIDATES = 1
HOST_CANDGEN = 2
NO_OVERLAP_INGEST = 4
COMPLETE_INTERSECTION = 8
MULTI_KERNEL = 16
MEM_HOST, MEM_DEVICE = 0, 1
PHASES = ["upload", "histogram", "bitset", "candgen", "count", "threshold", "total"]
STATUS = {0: "GPA_OK", 1: "GPA_ERR_INVALID", 2: "GPA_ERR_RANGE", 3: "GPA_ERR_OOM", 4: "GPA_ERR_CUDA",
          5: "GPA_ERR_NCCL", 6: "GPA_ERR_STATE"}


class GpaError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class _CSR(ctypes.Structure):
    _fields_ = [("n_tx", ctypes.c_uint64), ("offsets", ctypes.c_void_p), ("items", ctypes.c_void_p),
                ("n_items", ctypes.c_uint32), ("memory", ctypes.c_uint32)]


class _Options(ctypes.Structure):
    _fields_ = [("count_kernel", ctypes.c_uint32), ("flags", ctypes.c_uint32), ("stream", ctypes.c_void_p),
                ("device", ctypes.c_int32), ("max_k", ctypes.c_uint32), ("reserved", ctypes.c_uint32 * 3)]


class _LevelStats(ctypes.Structure):
    _fields_ = [("n_cand", ctypes.c_uint64), ("n_freq", ctypes.c_uint64), ("n_groups", ctypes.c_uint64),
                ("kernel", ctypes.c_uint32), ("launches", ctypes.c_uint32), ("count_ms", ctypes.c_double),
                ("allreduce_ms", ctypes.c_double), ("candgen_ms", ctypes.c_double), ("build_ms", ctypes.c_double),
                ("build_words", ctypes.c_uint64), ("setup_ms", ctypes.c_double), ("build_bytes", ctypes.c_uint64),
                ("count_bytes", ctypes.c_uint64)]


_LIB = None
# int fn(void* ctx, void* host_buf, uint64_t n, uint32_t dtype, uint32_t op)  (gpa_host_allreduce_fn)
_HOST_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32,
                            ctypes.c_uint32)
DT_U32, DT_U64 = 0, 1
OP_SUM, OP_MAX = 0, 1


def lib() -> ctypes.CDLL:
    """Load libgpapriori.so (built in-tree by ``make`` / ``__graft_entry__.build()``)."""
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `make` (no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH)
    vp, u32, u64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64
    P = ctypes.POINTER
    sig = {
        "gpa_last_error": (ctypes.c_char_p, []),
        "gpa_version": (ctypes.c_char_p, []),
        "gpa_kernel_launches": (ctypes.c_uint64, []),
        "gpa_options_default": (None, [P(_Options)]),
        "gpa_min_count": (u64, [u64, u64, u64]),
        "gpa_dist_unique_id": (ctypes.c_int, [ctypes.c_char_p]),
        "gpa_dist_create": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_char_p, P(vp)]),
        "gpa_dist_destroy": (ctypes.c_int, [vp]),
        "gpa_dist_info": (ctypes.c_int, [vp, P(ctypes.c_int), P(ctypes.c_int)]),
        "gpa_dist_create_host": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int, _HOST_FN, vp, P(vp)]),
        "gpa_dist_log": (ctypes.c_int, [vp, P(u64), u64, P(u64)]),
        "gpa_dist_set_timeout": (ctypes.c_int, [vp, ctypes.c_double]),
        "gpa_bitset_create": (ctypes.c_int, [P(_CSR), u32, vp, P(_Options), P(vp)]),
        "gpa_bitset_destroy": (ctypes.c_int, [vp]),
        "gpa_bitset_info": (ctypes.c_int, [vp, P(u64), P(u64), P(u32), P(u64)]),
        "gpa_bitset_item_counts": (ctypes.c_int, [vp, vp]),
        "gpa_bitset_rows": (ctypes.c_int, [vp, vp]),
        "gpa_bitset_export": (ctypes.c_int, [vp, vp]),
        "gpa_count": (ctypes.c_int, [vp, vp, u32, u64, u32, vp]),
        "gpa_mine": (ctypes.c_int, [P(_CSR), u64, vp, P(_Options), P(vp)]),
        "gpa_result_info": (ctypes.c_int, [vp, P(u64), P(u64)]),
        "gpa_result_count": (ctypes.c_int, [vp, P(u64), P(u32)]),
        "gpa_result_get": (ctypes.c_int, [vp, u64, P(P(u32)), P(u32), P(u32)]),
        "gpa_result_frequent": (ctypes.c_int, [vp, u32, P(u64), P(P(u32)), P(P(u32))]),
        "gpa_result_level": (ctypes.c_int, [vp, u32, P(u64), P(u64), P(P(u32)), P(P(u32))]),
        "gpa_result_n_levels": (ctypes.c_int, [vp, P(u32)]),
        "gpa_result_level_stats": (ctypes.c_int, [vp, u32, P(_LevelStats)]),
        "gpa_result_timing": (ctypes.c_int, [vp, ctypes.c_double * 7]),
        "gpa_result_destroy": (ctypes.c_int, [vp]),
        "gpa_rules_create": (ctypes.c_int, [vp, u64, u64, P(vp)]),
        "gpa_rules_arrays": (ctypes.c_int, [vp, P(u64), P(P(u32)), P(P(u32)), P(P(u32))]),
        "gpa_rules_destroy": (ctypes.c_int, [vp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


def _check(status: int) -> None:
    if status != 0:
        raise GpaError(status, lib().gpa_last_error().decode())


def version() -> str:
    return lib().gpa_version().decode()


def kernel_launches() -> int:
    """Kernels this library has launched in the process so far (gpa_kernel_launches)."""
    return int(lib().gpa_kernel_launches())


def min_count(n_tx: int, minsup) -> int:
    """max(1, ceil(minsup * n_tx)) with minsup an exact decimal (string) or Fraction (gpa_min_count)."""
    f = Fraction(minsup)
    return int(lib().gpa_min_count(int(n_tx), f.numerator, f.denominator))


@dataclass
class Options:
    count_kernel: int = KERNEL_AUTO
    keep_candidates: bool = False
    stream: int = 0          # cudaStream_t as an integer (e.g. torch.cuda.current_stream().cuda_stream); 0 = own
    device: int = -1
    max_k: int = 0
    host_candgen: bool = False   # join + prune on the host (reference path) instead of the device
    overlap_ingest: bool = True  # host input: chunked upload overlapped with histogram / bitset / pairs
    complete_intersection: bool = False   # k >= 3 by complete intersection (the paper's method), no lists
    multi_kernel: bool = False   # never the single-launch small-problem path (KERNEL_FUSED) under AUTO

    def _c(self) -> _Options:
        o = _Options()
        lib().gpa_options_default(ctypes.byref(o))
        o.count_kernel = self.count_kernel
        o.flags = ((KEEP_CANDIDATES if self.keep_candidates else 0) | (HOST_CANDGEN if self.host_candgen else 0)
                   | (0 if self.overlap_ingest else NO_OVERLAP_INGEST)
                   | (COMPLETE_INTERSECTION if self.complete_intersection else 0)
                   | (MULTI_KERNEL if self.multi_kernel else 0))
        o.stream = self.stream or None
        o.device = self.device
        o.max_k = self.max_k
        return o


def _is_torch(x) -> bool:
    return type(x).__module__.startswith("torch")


class _Input:
    """CSR marshalling: keeps the arrays alive while the C call runs."""

    def __init__(self, offsets, items, n_items: int):
        self.keep = []
        dev = _is_torch(offsets) and offsets.is_cuda
        if dev:
            assert _is_torch(items) and items.is_cuda, "offsets and items must both be CUDA tensors"
            assert offsets.element_size() == 8 and items.element_size() == 4
            offsets, items = offsets.contiguous(), items.contiguous()
            self.keep += [offsets, items]
            self.c = _CSR(offsets.numel() - 1, offsets.data_ptr(), items.data_ptr() if items.numel() else None,
                          int(n_items), MEM_DEVICE)
        else:
            if _is_torch(offsets):
                offsets, items = offsets.numpy(), items.numpy()
            o = np.ascontiguousarray(offsets).view(np.uint64) if np.asarray(offsets).dtype.itemsize == 8 else \
                np.ascontiguousarray(offsets, dtype=np.uint64)
            it = np.ascontiguousarray(items)
            it = it.view(np.uint32) if it.dtype.itemsize == 4 and it.dtype.kind in "iu" else it.astype(np.uint32)
            self.keep += [o, it]
            self.c = _CSR(len(o) - 1, o.ctypes.data, it.ctypes.data if it.size else None, int(n_items), MEM_HOST)


def _args(db, items, n_items):
    if items is None:  # a dataset object with .offsets/.items/.n_items
        return db.offsets, db.items, db.n_items
    return db, items, n_items


def torch_host_allreduce(arr: np.ndarray, op: str) -> None:
    """In-place all-reduce of a uint32 / uint64 host array over the current torch.distributed group
    (the host-staged transport's callback).  Unsigned semantics through torch's signed tensors:
    sums wrap in two's complement (bit-identical to the unsigned sum), max compares after flipping
    the sign bit."""
    import torch
    import torch.distributed as tdist
    t = torch.from_numpy(arr.view(np.int64) if arr.dtype == np.uint64 else arr.view(np.int32))
    if op == "max":
        sign = -2 ** 63 if arr.dtype == np.uint64 else -2 ** 31
        t ^= sign
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        t ^= sign
    else:
        tdist.all_reduce(t, op=tdist.ReduceOp.SUM)


class Dist:
    """Communicator over the ranks of a torch.distributed job: NCCL (one process per GPU), or the
    host-staged transport (gpa_dist_create_host) over any in-place host all-reduce."""

    def __init__(self, rank: int, world: int, device: int, unique_id: bytes | None = None, host_allreduce=None):
        h = ctypes.c_void_p()
        self._fn = None
        if host_allreduce is not None:
            def fn(_ctx, buf, n, dtype, op):
                try:
                    ct = ctypes.c_uint32 if dtype == DT_U32 else ctypes.c_uint64
                    arr = np.ctypeslib.as_array((ct * int(n)).from_address(buf))
                    host_allreduce(arr, "max" if op == OP_MAX else "sum")
                    return 0
                except Exception:   # reported to the library as a failed collective
                    import traceback
                    traceback.print_exc()
                    return 1
            self._fn = _HOST_FN(fn)   # must outlive every library call on this handle
            _check(lib().gpa_dist_create_host(rank, world, device, self._fn, None, ctypes.byref(h)))
        else:
            _check(lib().gpa_dist_create(rank, world, device, unique_id, ctypes.byref(h)))
        self.h, self.rank, self.world = h, rank, world

    @classmethod
    def host_from_torch(cls, device: int) -> "Dist":
        """Host-staged transport over the current torch.distributed group (e.g. gloo): lets several
        ranks share one GPU, which NCCL refuses."""
        import torch.distributed as tdist
        return cls(tdist.get_rank(), tdist.get_world_size(), device, host_allreduce=torch_host_allreduce)

    def log(self) -> list:
        """Every collective this handle issued, in order: (op, dtype, n) tuples (gpa_dist_log)."""
        n = ctypes.c_uint64()
        _check(lib().gpa_dist_log(self.h, None, 0, ctypes.byref(n)))
        buf = (ctypes.c_uint64 * max(n.value, 1))()
        _check(lib().gpa_dist_log(self.h, buf, n.value, ctypes.byref(n)))
        return [(int(v) >> 60, (int(v) >> 56) & 15, int(v) & ((1 << 56) - 1)) for v in buf[: n.value]]

    def set_timeout(self, seconds: float) -> None:
        _check(lib().gpa_dist_set_timeout(self.h, float(seconds)))

    @staticmethod
    def unique_id() -> bytes:
        buf = ctypes.create_string_buffer(128)
        _check(lib().gpa_dist_unique_id(buf))
        return buf.raw

    @classmethod
    def from_torch(cls, device: int) -> "Dist":
        """Rank 0 creates the NCCL id; torch.distributed broadcasts its 128 bytes."""
        import torch
        import torch.distributed as tdist
        rank, world = tdist.get_rank(), tdist.get_world_size()
        uid = cls.unique_id() if rank == 0 else bytes(128)
        t = torch.tensor(list(uid), dtype=torch.uint8)
        if tdist.get_backend() == "nccl":
            t = t.cuda(device)
        tdist.broadcast(t, 0)
        return cls(rank, world, device, bytes(t.cpu().tolist()))

    def close(self):
        if self.h:
            _check(lib().gpa_dist_destroy(self.h))
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Bitset:
    """The static bitset of a transaction database on the GPU (gpa_bitset_create)."""

    def __init__(self, db, items=None, n_items=None, row_min_count: int = 1, dist: Dist | None = None,
                 options: Options | None = None):
        off, it, ni = _args(db, items, n_items)
        inp = _Input(off, it, ni)
        opt = (options or Options())._c()
        h = ctypes.c_void_p()
        _check(lib().gpa_bitset_create(ctypes.byref(inp.c), row_min_count, dist.h if dist else None,
                                       ctypes.byref(opt), ctypes.byref(h)))
        self.h, self.n_items = h, int(ni)
        a, b, c, d = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint32(), ctypes.c_uint64()
        _check(lib().gpa_bitset_info(h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c), ctypes.byref(d)))
        self.n_tx_local, self.n_tx, self.n_rows, self.row_pitch_bytes = a.value, b.value, c.value, d.value

    def item_counts(self) -> np.ndarray:
        out = np.zeros(max(self.n_items, 1), dtype=np.uint32)
        _check(lib().gpa_bitset_item_counts(self.h, out.ctypes.data))
        return out[: self.n_items]

    def rows(self) -> np.ndarray:
        out = np.zeros(max(self.n_rows, 1), dtype=np.uint32)
        _check(lib().gpa_bitset_rows(self.h, out.ctypes.data))
        return out[: self.n_rows]

    def export(self) -> np.ndarray:
        """(n_rows, row_pitch_bytes/4) uint32 words of this rank's rows (bit t%32 of word t/32)."""
        out = np.zeros((max(self.n_rows, 1), self.row_pitch_bytes // 4), dtype=np.uint32)
        _check(lib().gpa_bitset_export(self.h, out.ctypes.data))
        return out[: self.n_rows]

    def count(self, cand, kernel: int = KERNEL_AUTO) -> np.ndarray:
        """Supports of candidates ((M, k) original item ids, rows strictly increasing)."""
        c = np.ascontiguousarray(cand, dtype=np.uint32)
        if c.ndim != 2:
            raise ValueError("cand must be (M, k)")
        M, k = c.shape
        out = np.zeros(max(M, 1), dtype=np.uint32)
        _check(lib().gpa_count(self.h, c.ctypes.data if M else None, k, M, kernel, out.ctypes.data))
        return out[:M]

    def close(self):
        if self.h:
            _check(lib().gpa_bitset_destroy(self.h))
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


@dataclass
class Level:
    k: int
    n_cand: int
    n_freq: int
    freq_items: np.ndarray        # (n_freq, k) item ids, lexicographic
    freq_support: np.ndarray      # (n_freq,)
    cand: np.ndarray | None       # (n_cand, k) with keep_candidates
    counts: np.ndarray | None     # (n_cand,)  with keep_candidates
    stats: dict = field(default_factory=dict)


@dataclass
class MineResult:
    n_tx: int
    min_count: int
    levels: list
    timing_ms: dict
    _owner: object = None   # the library's result handle (kept for rules())

    def rules(self, minconf: str | Fraction | float = "0.5") -> "Rules":
        """Association rules A => X \\ A with supp(X) / supp(A) >= minconf (gpa_rules_create; exact
        rational comparison: minconf is parsed as a decimal string / Fraction)."""
        f = Fraction(str(minconf)) if not isinstance(minconf, Fraction) else minconf
        L = lib()
        h = ctypes.c_void_p()
        _check(L.gpa_rules_create(self._owner.h, f.numerator, f.denominator, ctypes.byref(h)))
        owner = _ResultOwner(h, L.gpa_rules_destroy)   # the arrays below view the rules' memory
        n = ctypes.c_uint64()
        px, pm, ps = (ctypes.POINTER(ctypes.c_uint32)() for _ in range(3))
        _check(L.gpa_rules_arrays(h, ctypes.byref(n), ctypes.byref(px), ctypes.byref(pm), ctypes.byref(ps)))
        return Rules(self, _view(owner, px, n.value, (n.value,)), _view(owner, pm, n.value, (n.value,)),
                     _view(owner, ps, n.value, (n.value,)))

    def frequent(self, k: int | None = None):
        """F as {itemset tuple: support} (k=None), or the (items, supports) arrays of F_k."""
        if k is not None:
            lv = self.levels[k - 1] if k <= len(self.levels) else None
            if lv is None:
                return np.zeros((0, k), np.uint32), np.zeros(0, np.uint32)
            return lv.freq_items, lv.freq_support
        out = {}
        for lv in self.levels:
            for row, s in zip(lv.freq_items.tolist(), lv.freq_support.tolist()):
                out[tuple(row)] = s
        return out

    def level_map(self, k: int) -> dict:
        lv = self.levels[k - 1]
        return {tuple(r): int(c) for r, c in zip(lv.cand.tolist(), lv.counts.tolist())}

    @property
    def cand_tx(self) -> int:
        """sum_{k>=2} |C_k| * N: the candidate x transaction work counted on the GPU."""
        return sum(lv.n_cand for lv in self.levels[1:]) * self.n_tx

    @property
    def count_ms(self) -> float:
        return sum(lv.stats.get("count_ms", 0.0) for lv in self.levels[1:])


@dataclass
class Rules:
    """Association rules of a MineResult: rule j is (X = itemset number itemset[j] in canonical
    order, antecedent = X's items selected by the bits of antecedent_mask[j], supp(A) =
    antecedent_support[j])."""
    result: "MineResult"
    itemset: np.ndarray
    antecedent_mask: np.ndarray
    antecedent_support: np.ndarray

    def __len__(self):
        return len(self.itemset)

    def as_dict(self) -> dict:
        """{(antecedent tuple, consequent tuple): (supp(X), supp(A))}."""
        flat = [(tuple(r), int(s)) for lv in self.result.levels for r, s in zip(lv.freq_items.tolist(),
                                                                               lv.freq_support.tolist())]
        out = {}
        for x, m, sa in zip(self.itemset.tolist(), self.antecedent_mask.tolist(), self.antecedent_support.tolist()):
            X, sx = flat[x]
            A = tuple(v for q, v in enumerate(X) if m >> q & 1)
            B = tuple(v for q, v in enumerate(X) if not m >> q & 1)
            out[(A, B)] = (sx, sa)
        return out


def _arr(ptr, n, shape):
    if n == 0 or not ptr:
        return np.zeros(shape, dtype=np.uint32)
    return np.ctypeslib.as_array(ptr, (n,)).copy().reshape(shape)


class _ResultOwner:
    """Owns a library handle (gpa_result, or gpa_rules with its destroy function); arrays viewing
    its memory keep it alive (freed with the last one)."""

    def __init__(self, h, destroy=None):
        self.h = h
        self.destroy = destroy

    def __del__(self):
        if self.h:
            try:
                (self.destroy or lib().gpa_result_destroy)(self.h)
            except Exception:   # interpreter shutdown
                pass
            self.h = None


def _view(owner, ptr, n, shape):
    """Zero-copy uint32 view of library-owned result memory (kept alive through ``owner``)."""
    if n == 0 or not ptr:
        return np.zeros(shape, dtype=np.uint32)
    buf = (ctypes.c_uint32 * n).from_address(ctypes.addressof(ptr.contents))
    buf._gpa_owner = owner
    return np.frombuffer(buf, dtype=np.uint32).reshape(shape)


def mine(db, items=None, n_items=None, min_count: int = 1, dist: Dist | None = None,
         options: Options | None = None, keep_candidates: bool | None = None) -> MineResult:
    """Level-wise mining with GPU support counting (gpa_mine)."""
    off, it, ni = _args(db, items, n_items)
    inp = _Input(off, it, ni)
    o = options or Options()
    if keep_candidates is not None:
        import dataclasses
        o = dataclasses.replace(o, keep_candidates=keep_candidates)
    copt = o._c()
    L = lib()
    h = ctypes.c_void_p()
    _check(L.gpa_mine(ctypes.byref(inp.c), int(min_count), dist.h if dist else None, ctypes.byref(copt),
                      ctypes.byref(h)))
    owner = _ResultOwner(h)   # the result's arrays below are views of its memory (no copy of F)
    try:
        nl = ctypes.c_uint32()
        _check(L.gpa_result_n_levels(h, ctypes.byref(nl)))
        levels = []
        n_tx = 0
        for k in range(1, nl.value + 1):
            nc, nf = ctypes.c_uint64(), ctypes.c_uint64()
            cp, cc = ctypes.POINTER(ctypes.c_uint32)(), ctypes.POINTER(ctypes.c_uint32)()
            _check(L.gpa_result_level(h, k, ctypes.byref(nc), ctypes.byref(nf), ctypes.byref(cp), ctypes.byref(cc)))
            n2 = ctypes.c_uint64()
            fi, fs = ctypes.POINTER(ctypes.c_uint32)(), ctypes.POINTER(ctypes.c_uint32)()
            _check(L.gpa_result_frequent(h, k, ctypes.byref(n2), ctypes.byref(fi), ctypes.byref(fs)))
            st = _LevelStats()
            _check(L.gpa_result_level_stats(h, k, ctypes.byref(st)))
            stats = {f: getattr(st, f) for f, _ in _LevelStats._fields_}
            stats["kernel_name"] = KERNEL_NAMES.get(st.kernel, "?")
            kept = bool(cp)
            levels.append(Level(k, nc.value, nf.value, _view(owner, fi, nf.value * k, (nf.value, k)),
                                _view(owner, fs, nf.value, (nf.value,)),
                                _view(owner, cp, nc.value * k, (nc.value, k)) if kept else None,
                                _view(owner, cc, nc.value, (nc.value,)) if kept else None, stats))
        ntx, mc = ctypes.c_uint64(), ctypes.c_uint64()
        _check(L.gpa_result_info(h, ctypes.byref(ntx), ctypes.byref(mc)))
        n_tx = ntx.value
        tm = (ctypes.c_double * 7)()
        _check(L.gpa_result_timing(h, tm))
        timing = {PHASES[i]: tm[i] for i in range(7)}
    except BaseException:
        del owner
        raise
    return MineResult(n_tx, int(min_count), levels, timing, owner)
