"""Thin ctypes binding of libbzk.so (include/bzk.h) -- argument marshalling only.

Every step of the prover runs in the CUDA library; if ``libbzk.so`` is missing or cannot be
loaded this module raises -- there is no CPU fallback.  Function names follow the C ABI
(``bzk_create``, ``bzk_prove``, ...); :class:`Prover` is a small convenience wrapper that
allocates torch output tensors.

Buffers are passed as raw pointers: torch tensors (device or pinned host) via ``data_ptr()``,
numpy arrays via ``ctypes``.  Field elements are 4 x 64-bit little-endian limbs; torch has no
full uint64 support, so tensors are int64 holding the same bits.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# BZK_LIB overrides the library path (A/B experiments with alternative builds)
LIB_PATH = os.environ.get("BZK_LIB", os.path.join(HERE, "libbzk.so"))

BZK_OK, BZK_EINVAL, BZK_ENOMEM, BZK_ECUDA, BZK_ENONCANON, BZK_EUNSUPPORTED = range(6)
BZK_ORDER_LSB, BZK_ORDER_MSB = 0, 1
BZK_MEM_DEVICE, BZK_MEM_HOST = 0, 1
BZK_F_PRESERVE_INPUT, BZK_F_VALIDATE, BZK_F_SYNC, BZK_F_GRAPH, BZK_F_GIVEN_CHALLENGES = 1, 2, 4, 8, 16
BZK_F_FIELD_GOLDILOCKS = 32
BZK_F_SEEDS_DEVICE = 64
BZK_PROF_KINDS = 12
PROF_KIND_NAMES = ["round1_eval", "fused_fold_eval", "tail", "transcript_init", "validate", "h2d_copy",
                   "merkle_stage", "d2h_copy", "encoder_spmv", "multi_round", "small_cluster",
                   "multi_round_tc"]
BZK_MERKLE_COMPRESS, BZK_MERKLE_SHA256 = 0, 1

EXPORTS = ["bzk_create", "bzk_destroy", "bzk_workspace_size", "bzk_prove", "bzk_prove_ragged", "bzk_sync",
           "bzk_strerror", "bzk_last_error", "bzk_generate", "bzk_profile_enable", "bzk_profile_read",
           "bzk_launch_count", "bzk_debug_field", "bzk_debug_sha256", "bzk_debug_bench", "bzk_version",
           "bzk_merkle", "bzk_generate_blocks", "bzk_encoder_create", "bzk_encoder_destroy", "bzk_encode",
           "bzk_debug_gl", "bzk_commit_prove"]


class BzkError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"bzk status {status} ({_strerror(status)}){': ' + detail if detail else ''}")


class bzk_batch(ctypes.Structure):
    _fields_ = [("num_vars", ctypes.c_uint32), ("degree", ctypes.c_uint32), ("order", ctypes.c_uint32),
                ("flags", ctypes.c_uint32), ("batch", ctypes.c_uint64), ("first_index", ctypes.c_uint64),
                ("seed", ctypes.c_void_p), ("tables", ctypes.c_void_p), ("tables_mem", ctypes.c_uint32),
                ("outputs_mem", ctypes.c_uint32), ("round_evals", ctypes.c_void_p),
                ("challenges", ctypes.c_void_p), ("final_evals", ctypes.c_void_p), ("claims", ctypes.c_void_p)]


class bzk_merkle_batch(ctypes.Structure):
    _fields_ = [("log_blocks", ctypes.c_uint32), ("hash", ctypes.c_uint32), ("flags", ctypes.c_uint32),
                ("blocks_mem", ctypes.c_uint32), ("batch", ctypes.c_uint64), ("blocks", ctypes.c_void_p),
                ("outputs_mem", ctypes.c_uint32), ("reserved", ctypes.c_uint32), ("roots", ctypes.c_void_p),
                ("nodes", ctypes.c_void_p)]


class bzk_csr(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_uint32), ("cols", ctypes.c_uint32), ("nnz", ctypes.c_uint64),
                ("row_ptr", ctypes.c_void_p), ("col", ctypes.c_void_p), ("val", ctypes.c_void_p)]


class bzk_commit(ctypes.Structure):
    _fields_ = [("segments", ctypes.c_uint32), ("hash", ctypes.c_uint32), ("codes", ctypes.c_void_p),
                ("roots", ctypes.c_void_p), ("nodes", ctypes.c_void_p), ("final_roots", ctypes.c_void_p)]


class bzk_code(ctypes.Structure):
    _fields_ = [("log_n", ctypes.c_uint32), ("levels", ctypes.c_uint32), ("A", ctypes.c_void_p),
                ("B", ctypes.c_void_p), ("G0", ctypes.c_void_p)]


_lib = None


def lib():
    """Load libbzk.so (raises if absent: no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run python -m paper_conf_asplos_lucw0cz25_b200.build "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        L.bzk_create.argtypes = [i32, ctypes.c_size_t, ctypes.POINTER(vp)]
        L.bzk_destroy.argtypes = [vp]
        L.bzk_destroy.restype = None
        L.bzk_workspace_size.argtypes = [vp, ctypes.POINTER(bzk_batch), ctypes.POINTER(ctypes.c_size_t)]
        L.bzk_prove.argtypes = [vp, ctypes.POINTER(bzk_batch), vp]
        L.bzk_prove_ragged.argtypes = [vp, ctypes.POINTER(bzk_batch), ctypes.c_size_t, vp]
        L.bzk_sync.argtypes = [vp]
        L.bzk_strerror.argtypes = [i32]
        L.bzk_strerror.restype = ctypes.c_char_p
        L.bzk_last_error.argtypes = [vp]
        L.bzk_last_error.restype = ctypes.c_char_p
        L.bzk_generate.argtypes = [vp, u64, u32, u32, u64, u32, u64, vp]
        L.bzk_profile_enable.argtypes = [vp, i32]
        L.bzk_profile_read.argtypes = [vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(u64), i32]
        L.bzk_launch_count.argtypes = [vp, i32]
        L.bzk_launch_count.restype = u64
        L.bzk_debug_field.argtypes = [i32, u64, vp, vp, vp, vp]
        L.bzk_debug_sha256.argtypes = [vp, u32, u64, vp, vp]
        L.bzk_debug_gl.argtypes = [i32, u64, vp, vp, vp, vp]
        L.bzk_debug_bench.argtypes = [i32, u32, ctypes.POINTER(ctypes.c_double), vp]
        L.bzk_version.restype = ctypes.c_char_p
        L.bzk_merkle.argtypes = [vp, ctypes.POINTER(bzk_merkle_batch), vp]
        L.bzk_generate_blocks.argtypes = [vp, u64, u32, u64, u64, vp]
        L.bzk_encoder_create.argtypes = [vp, ctypes.POINTER(bzk_code), ctypes.POINTER(vp)]
        L.bzk_encoder_destroy.argtypes = [vp]
        L.bzk_encoder_destroy.restype = None
        L.bzk_encode.argtypes = [vp, vp, vp, u64, u32, u32, vp]
        L.bzk_commit_prove.argtypes = [vp, vp, ctypes.POINTER(bzk_commit), ctypes.POINTER(bzk_batch), vp]
        for name in ("bzk_create", "bzk_workspace_size", "bzk_prove", "bzk_prove_ragged", "bzk_sync",
                     "bzk_generate", "bzk_profile_enable", "bzk_profile_read", "bzk_debug_field",
                     "bzk_debug_sha256", "bzk_debug_bench", "bzk_debug_gl", "bzk_merkle", "bzk_generate_blocks",
                     "bzk_encoder_create", "bzk_encode", "bzk_commit_prove"):
            getattr(L, name).restype = i32
        _lib = L
    return _lib


def _strerror(s: int) -> str:
    try:
        return lib().bzk_strerror(s).decode()
    except Exception:  # noqa: BLE001
        return "?"


def _check(status: int, ctx=None):
    if status != BZK_OK:
        detail = lib().bzk_last_error(ctx).decode() if ctx else ""
        raise BzkError(status, detail)


def ptr(x) -> int | None:
    """Raw address of a torch tensor / numpy array / int (None passes through)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    raise TypeError(type(x))


def _stream_handle(stream) -> int | None:
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except ImportError:
            pass
        return None
    if hasattr(stream, "cuda_stream"):
        return stream.cuda_stream
    return int(stream)


# ---------------------------------------------------------------- C-ABI names

def bzk_create(device: int = 0, workspace_limit: int = 0):
    h = ctypes.c_void_p()
    _check(lib().bzk_create(device, workspace_limit, ctypes.byref(h)))
    return h


def bzk_destroy(ctx) -> None:
    lib().bzk_destroy(ctx)


def make_batch(k, d, order, flags, batch, first_index, seed_buf, tables, tables_mem, outputs_mem, round_evals,
               challenges, final_evals, claims) -> bzk_batch:
    seed = ctypes.c_void_p(seed_buf) if isinstance(seed_buf, int) else ctypes.cast(seed_buf, ctypes.c_void_p)
    return bzk_batch(k, d, order, flags, batch, first_index, seed, ptr(tables),
                     tables_mem, outputs_mem, ptr(round_evals), ptr(challenges), ptr(final_evals), ptr(claims))


def bzk_prove(ctx, b: bzk_batch, stream=None) -> None:
    _check(lib().bzk_prove(ctx, ctypes.byref(b), _stream_handle(stream)), ctx)


def bzk_prove_ragged(ctx, jobs: list[bzk_batch], stream=None) -> None:
    arr = (bzk_batch * len(jobs))(*jobs)
    _check(lib().bzk_prove_ragged(ctx, arr, len(jobs), _stream_handle(stream)), ctx)


def bzk_workspace_size(ctx, b: bzk_batch) -> int:
    n = ctypes.c_size_t()
    _check(lib().bzk_workspace_size(ctx, ctypes.byref(b), ctypes.byref(n)), ctx)
    return n.value


def bzk_sync(ctx) -> None:
    _check(lib().bzk_sync(ctx), ctx)


def bzk_generate(dst, batch, d, k, first_index=0, dist=0, data_seed=None, stream=None) -> None:
    from .inputs import DATA_SEED, DISTS
    if isinstance(dist, str):
        dist = DISTS[dist]
    _check(lib().bzk_generate(ptr(dst), batch, d, k, first_index, dist,
                              DATA_SEED if data_seed is None else data_seed, _stream_handle(stream)))


def bzk_merkle(ctx, b: bzk_merkle_batch, stream=None) -> None:
    _check(lib().bzk_merkle(ctx, ctypes.byref(b), _stream_handle(stream)), ctx)


def bzk_generate_blocks(dst, batch, n, first_index=0, data_seed=None, stream=None) -> None:
    from .inputs import MERKLE_DATA_SEED
    _check(lib().bzk_generate_blocks(ptr(dst), batch, n, first_index,
                                     MERKLE_DATA_SEED if data_seed is None else data_seed, _stream_handle(stream)))


def _csr_struct(m: dict) -> bzk_csr:
    for k_ in ("row_ptr", "col", "val"):
        assert m[k_].flags["C_CONTIGUOUS"]
    return bzk_csr(m["rows"], m["cols"], int(m["row_ptr"][-1]), m["row_ptr"].ctypes.data, m["col"].ctypes.data,
                   m["val"].ctypes.data)


def bzk_encoder_create(ctx, code: dict):
    """code: the dict of inputs.gen_code (host CSR arrays).  Returns an opaque encoder handle."""
    L = code["levels"]
    A = (bzk_csr * max(1, L))(*[_csr_struct(a) for a in code["A"]])
    B = (bzk_csr * max(1, L))(*[_csr_struct(b) for b in code["B"]])
    G0 = _csr_struct(code["G0"])
    c = bzk_code(code["log_n"], L, ctypes.addressof(A), ctypes.addressof(B), ctypes.addressof(G0))
    h = ctypes.c_void_p()
    _check(lib().bzk_encoder_create(ctx, ctypes.byref(c), ctypes.byref(h)), ctx)
    return h


def bzk_encoder_destroy(enc) -> None:
    lib().bzk_encoder_destroy(enc)


def bzk_encode(ctx, enc, codes, batch: int, codes_mem: int = BZK_MEM_DEVICE, flags: int = 0, stream=None) -> None:
    _check(lib().bzk_encode(ctx, enc, ptr(codes), batch, codes_mem, flags, _stream_handle(stream)), ctx)


def bzk_commit_prove(ctx, enc, commit: bzk_commit, sumcheck: bzk_batch, stream=None) -> None:
    _check(lib().bzk_commit_prove(ctx, enc, ctypes.byref(commit), ctypes.byref(sumcheck), _stream_handle(stream)), ctx)


def bzk_profile_enable(ctx, on: bool) -> None:
    _check(lib().bzk_profile_enable(ctx, int(on)), ctx)


def bzk_profile_read(ctx, reset: bool = True) -> dict:
    ms = (ctypes.c_double * BZK_PROF_KINDS)()
    cnt = (ctypes.c_uint64 * BZK_PROF_KINDS)()
    _check(lib().bzk_profile_read(ctx, ms, cnt, int(reset)), ctx)
    return {PROF_KIND_NAMES[i]: (ms[i], cnt[i]) for i in range(BZK_PROF_KINDS)}


def bzk_launch_count(ctx, reset: bool = False) -> int:
    return int(lib().bzk_launch_count(ctx, int(reset)))


def bzk_debug_field(op: int, n: int, a, b, out, stream=None) -> None:
    _check(lib().bzk_debug_field(op, n, ptr(a), ptr(b), ptr(out), _stream_handle(stream)))


def bzk_debug_gl(op: int, n: int, a, b, out, stream=None) -> None:
    _check(lib().bzk_debug_gl(op, n, ptr(a), ptr(b), ptr(out), _stream_handle(stream)))


def bzk_debug_sha256(msgs, msg_len: int, n: int, out, stream=None) -> None:
    _check(lib().bzk_debug_sha256(ptr(msgs), msg_len, n, ptr(out), _stream_handle(stream)))


def bzk_debug_bench(kind: int, iters: int = 4096, stream=None) -> float:
    """ops per SM per clock: kind 0 IMAD, 1 IMAD.WIDE, 2 reference mont_mul, 3 hot-path mont_mul."""
    r = ctypes.c_double()
    _check(lib().bzk_debug_bench(kind, iters, ctypes.byref(r), _stream_handle(stream)))
    return r.value


def bzk_version() -> str:
    return lib().bzk_version().decode()


# ---------------------------------------------------------------- convenience

class Prover:
    """Owns a bzk context; proves batches held in torch tensors (device or pinned host)."""

    def __init__(self, device: int = 0, workspace_limit: int = 0):
        self.device = device
        self.ctx = bzk_create(device, workspace_limit)
        self._seed_bufs = []

    def close(self):
        if self.ctx:
            bzk_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    @staticmethod
    def alloc_outputs(B, k, d, device="cuda", pin=False):
        import torch
        kw = dict(dtype=torch.int64, device=device)
        if device == "cpu" and pin:
            kw["pin_memory"] = True
        return {"round_evals": torch.empty((B, k, d + 1, 4), **kw),
                "challenges": torch.empty((B, k, 4), **kw),
                "final_evals": torch.empty((B, d, 4), **kw),
                "claims": torch.empty((B, 4), **kw)}

    @staticmethod
    def alloc_outputs_gl(B, k, d, device="cuda", pin=False):
        """Output tensors for BZK_F_FIELD_GOLDILOCKS (one 64-bit word per element)."""
        import torch
        kw = dict(dtype=torch.int64, device=device)
        if device == "cpu" and pin:
            kw["pin_memory"] = True
        return {"round_evals": torch.empty((B, k, d + 1), **kw), "challenges": torch.empty((B, k), **kw),
                "final_evals": torch.empty((B, d), **kw), "claims": torch.empty((B,), **kw)}

    def batch(self, tables, k, d, order=0, seed=None, first_index=0, flags=0, out=None, batch=None):
        from .inputs import DEFAULT_SEED
        seed = DEFAULT_SEED if seed is None else seed
        assert len(seed) == 32
        sb = ctypes.create_string_buffer(bytes(seed), 32)
        self._seed_bufs = [sb]
        B = batch if batch is not None else tables.shape[0]
        tables_host = hasattr(tables, "is_cuda") and not tables.is_cuda
        out_host = hasattr(out["final_evals"], "is_cuda") and not out["final_evals"].is_cuda
        return make_batch(k, d, order, flags, B, first_index, sb, tables,
                          BZK_MEM_HOST if tables_host else BZK_MEM_DEVICE,
                          BZK_MEM_HOST if out_host else BZK_MEM_DEVICE,
                          out["round_evals"], out["challenges"], out["final_evals"], out["claims"])

    def prove(self, tables, k, d, order=0, seed=None, first_index=0, flags=0, out=None, stream=None):
        """tables: int64 tensor [B][d][2^k][4]. Returns the output dict (torch tensors)."""
        B = tables.shape[0]
        if out is None:
            alloc = self.alloc_outputs_gl if flags & BZK_F_FIELD_GOLDILOCKS else self.alloc_outputs
            out = alloc(B, k, d, device="cuda" if tables.is_cuda else "cpu", pin=not tables.is_cuda)
        b = self.batch(tables, k, d, order, seed, first_index, flags, out)
        bzk_prove(self.ctx, b, stream)
        return out

    def sync(self):
        bzk_sync(self.ctx)


class MerkleBuilder:
    """Owns a bzk context; builds batches of Merkle trees held in torch tensors (device or pinned host).

    blocks: uint8 tensor [B][2^n][64].  Returns (roots uint8 [B][32], nodes uint8 [B][2^(n+1)-1][32] or None).
    """

    def __init__(self, device: int = 0, workspace_limit: int = 0, ctx=None):
        self.device = device
        self._own = ctx is None
        self.ctx = bzk_create(device, workspace_limit) if ctx is None else ctx

    def close(self):
        if self.ctx and self._own:
            bzk_destroy(self.ctx)
        self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    @staticmethod
    def batch(blocks, n, hash_mode=BZK_MERKLE_COMPRESS, roots=None, nodes=None, flags=0, batch=None):
        B = batch if batch is not None else blocks.shape[0]
        host_in = hasattr(blocks, "is_cuda") and not blocks.is_cuda
        host_out = hasattr(roots, "is_cuda") and not roots.is_cuda
        return bzk_merkle_batch(n, hash_mode, flags, BZK_MEM_HOST if host_in else BZK_MEM_DEVICE, B, ptr(blocks),
                                BZK_MEM_HOST if host_out else BZK_MEM_DEVICE, 0, ptr(roots), ptr(nodes))

    def build(self, blocks, n, hash_mode=BZK_MERKLE_COMPRESS, with_nodes=True, roots=None, nodes=None,
              flags=0, stream=None):
        import torch
        B = blocks.shape[0]
        dev = "cuda" if blocks.is_cuda else "cpu"
        pin = dev == "cpu"
        if roots is None:
            roots = torch.empty((B, 32), dtype=torch.uint8, device=dev, pin_memory=pin)
        if with_nodes and nodes is None:
            nodes = torch.empty((B, (2 << n) - 1, 32), dtype=torch.uint8, device=dev, pin_memory=pin)
        b = self.batch(blocks, n, hash_mode, roots, nodes if with_nodes else None, flags)
        bzk_merkle(self.ctx, b, stream)
        return roots, (nodes if with_nodes else None)


class Encoder:
    """Linear-time encoder (NEXT-4) for one code (graphs from inputs.gen_code); encodes batches in place.

    codes: int64 tensor [B][2n][4] (device, or pinned host) whose first n elements per row are the
    messages; after encode() each row is its codeword.
    """

    def __init__(self, code: dict, device: int = 0, ctx=None, workspace_limit: int = 0):
        self.device = device
        self._own = ctx is None
        self.ctx = bzk_create(device, workspace_limit) if ctx is None else ctx
        self.log_n = code["log_n"]
        self.enc = bzk_encoder_create(self.ctx, code)

    def close(self):
        if getattr(self, "enc", None):
            bzk_encoder_destroy(self.enc)
            self.enc = None
        if self.ctx and self._own:
            bzk_destroy(self.ctx)
        self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def encode(self, codes, flags: int = 0, stream=None):
        host = hasattr(codes, "is_cuda") and not codes.is_cuda
        bzk_encode(self.ctx, self.enc, codes, codes.shape[0], BZK_MEM_HOST if host else BZK_MEM_DEVICE, flags, stream)
        return codes
