"""Thin ctypes binding of the C ABI in include/apt.h (argument marshalling only).

Every step of the hot path runs in libapt.so's sm_100a kernels; this module
never computes anything itself and raises if the library is missing.  Names
mirror the C functions (``apt_sample`` -> ``Ctx.sample`` etc.).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libapt.so")

APT_OK, APT_E_INVALID, APT_E_OOM, APT_E_CUDA, APT_E_COMM, APT_E_UNSUPPORTED, APT_E_STATE, APT_E_DEVICE_ASSERT = range(8)
GDP, NFP, SNP, DNP, AUTO = range(5)
STRATEGY = {"GDP": GDP, "NFP": NFP, "SNP": SNP, "DNP": DNP, "AUTO": AUTO}
F32, BF16 = 0, 1
DTYPE = {"f32": F32, "bf16": BF16}
MAX_LAYERS, MAX_RANKS = 4, 8
READ = {"seeds": 0, "dst": 1, "Z": 2, "H": 3, "dW": 4, "db": 5, "G": 6, "dA": 7}


class AptError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"apt status {status}: {msg}")
        self.status = status


class BlockView(C.Structure):
    _fields_ = [("n_dst", C.c_int64), ("n_src", C.c_int64), ("n_edges", C.c_int64),
                ("dst_ids", C.c_void_p), ("src_ids", C.c_void_p), ("indptr", C.c_void_p), ("indices", C.c_void_p)]


class ModelDesc(C.Structure):
    _fields_ = [("n_layers", C.c_int), ("dims", C.c_int * (MAX_LAYERS + 1)), ("fanouts", C.c_int * MAX_LAYERS),
                ("batch", C.c_int), ("dtype", C.c_int), ("lr", C.c_float), ("sample_seed", C.c_uint64),
                ("feat_seed", C.c_uint64), ("gat_heads", C.c_int)]


_A4 = (C.c_int64 * MAX_RANKS) * 4
_D4 = (C.c_double * MAX_RANKS) * 4


class PlanStats(C.Structure):
    _fields_ = [("world", C.c_int), ("steps", C.c_int64), ("n_d", _A4), ("n_vs", C.c_int64 * MAX_RANKS),
                ("n_vd", C.c_int64 * MAX_RANKS), ("rows_local", _A4), ("rows_peer", _A4),
                ("feat_bytes_local", _A4), ("feat_bytes_peer", _A4), ("graph_bytes", _A4),
                ("hidden_bytes_fwd", _A4), ("hidden_bytes_bwd", _A4), ("n_calls", _A4),
                ("t_build_s", _D4), ("t_train_s", C.c_double), ("rows_host", _A4), ("feat_bytes_host", _A4),
                ("gat_heads", C.c_int), ("attn_bytes", _A4), ("attn_feat_bytes", _A4), ("t_resample_s", _D4),
                ("t_dryrun_s", C.c_double)]


class FstoreOpts(C.Structure):
    _fields_ = [("hbm_frac", C.c_double), ("cache_rows", C.c_int64), ("hot_ids", C.c_void_p),
                ("cache_rule", C.c_int), ("counts", C.c_void_p), ("cache_budget_rows", C.c_int64)]


class BwProfile(C.Structure):
    _fields_ = [("world", C.c_int), ("alpha_s", C.c_double * 8), ("beta_Bps", C.c_double * 8),
                ("measured", C.c_int * 8)]


_lib = None

# int (*apt_allgather_fn)(const void* send, void* recv, size_t bytes, void* user)
ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p)


def make_exchange(dist, group=None):
    """Bootstrap all-gather for a job of one process per GPU, on torch.distributed
    (any backend).  Plumbing only: the library calls it while creating objects to
    swap CUDA-IPC handles, never on the step path."""
    world = dist.get_world_size(group)

    @ALLGATHER_FN
    def fn(send, recv, nbytes, user):
        try:
            out = [None] * world
            dist.all_gather_object(out, C.string_at(send, nbytes), group=group)
            blob = b"".join(out)
            if len(blob) != nbytes * world:
                return 2
            C.memmove(recv, blob, len(blob))
            return 0
        except Exception:
            return 1
    return fn


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise AptError(-1, f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        vp, i64, i32, u64, st = C.c_void_p, C.c_int64, C.c_int, C.c_uint64, C.c_int
        sig = {
            "apt_ctx_create": [i32, i32, i32, vp, vp], "apt_ctx_destroy": [vp], "apt_ctx_sync": [vp],
            "apt_memcpy": [vp, vp, vp, C.c_size_t, i32],
            "apt_graph_load": [vp, i64, i64, vp, vp, vp, vp], "apt_graph_destroy": [vp],
            "apt_fstore_create": [vp, vp, i32, i32, i32, vp, u64, vp], "apt_fstore_destroy": [vp],
            "apt_fstore_create_tiered": [vp, vp, i32, i32, i32, vp, u64, vp, vp],
            "apt_sample": [vp, vp, vp, i64, vp, i32, u64, u64, vp], "apt_batch_block": [vp, i32, vp],
            "apt_batch_destroy": [vp], "apt_gather": [vp, vp, vp, i64, vp],
            "apt_aggregate": [vp, vp, vp, i32, i32, i64, vp, i64],
            "apt_aggregate_bwd": [vp, vp, vp, i32, i64, vp, i64],
            "apt_project": [vp, vp, i64, i32, vp, vp, i64, i32, i32, i32, vp, i64],
            "apt_weight_grad": [vp, vp, i64, vp, i64, i32, i64, i32, i32, vp, vp],
            "apt_trainer_create": [vp, vp, vp, vp, i32, vp, vp], "apt_trainer_destroy": [vp],
            "apt_trainer_set_params": [vp, i32, vp, vp], "apt_trainer_get_params": [vp, i32, i32, vp, vp],
            "apt_trainer_set_attention": [vp, vp, vp], "apt_trainer_get_attention": [vp, i32, vp, vp],
            "apt_trainer_set_epoch": [vp, vp, i64, u64], "apt_trainer_step": [vp, i64, i32],
            "apt_trainer_step_host": [vp, vp, i64, i64, i32, vp], "apt_trainer_loss": [vp, vp],
            "apt_trainer_step_host_pipelined": [vp, vp, i64, i64, i32, vp, vp],
            "apt_trainer_step_host_async": [vp, vp, i64, i64, i32, vp, vp],
            "apt_trainer_use_graph": [vp, i32], "apt_trainer_set_pipeline": [vp, i32], "apt_trainer_read": [vp, i32, i32, i32, vp, i64, vp, vp],
            "apt_trainer_phase_ms": [vp, vp, i32], "apt_trainer_agg_bytes": [vp, vp],
            "apt_partition": [i64, i64, vp, vp, i32, i32, u64, vp, vp],
            "apt_cache_sets": [i64, vp, vp, vp, i32, i32, vp, i64, vp, vp],
            "apt_dryrun": [vp, i64, vp], "apt_access_counts": [vp, i64, vp], "apt_hot_rows": [vp, i64, i64, vp], "apt_trainer_layer_fwd": [vp, i64], "apt_trainer_layer_bwd": [vp, vp, i64],
            "apt_layer_fwd": [vp, i32, vp, vp, vp, vp, i32, i32, vp, vp], "apt_layer_bwd": [vp, vp, vp, vp, vp],
            "apt_layer_saved_destroy": [vp], "apt_batch_group": [vp, vp, i32, vp], "apt_profile_links": [vp, vp], "apt_select_strategy": [vp, vp, vp, vp],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = st
        L.apt_last_error.argtypes = [vp]
        L.apt_last_error.restype = C.c_char_p
        L.apt_ctx_launches.argtypes = [vp]
        L.apt_ctx_launches.restype = C.c_int64
        L.apt_ctx_set_exchange.argtypes = [vp, ALLGATHER_FN, vp]
        L.apt_ctx_set_exchange.restype = st
        L.apt_exchange_selftest.argtypes = [i32, i32, ALLGATHER_FN, vp]
        L.apt_exchange_selftest.restype = st
        L.apt_selftest_div.argtypes = []
        L.apt_selftest_div.restype = C.c_int64
        L.apt_selftest_sort.argtypes = [i64, u64, i32]
        L.apt_selftest_sort.restype = C.c_int64
        L.apt_selftest_gemm.argtypes = [i32, i32, i32, i64, i32, i64, i32]
        L.apt_selftest_gemm.restype = C.c_double
        L.apt_trainer_steps_per_epoch.argtypes = [vp]
        L.apt_trainer_steps_per_epoch.restype = C.c_int64
        _lib = L
    return _lib


def _ptr(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    if hasattr(a, "data_ptr"):          # torch tensor (device memory / pinned host)
        return a.data_ptr()
    return a


def check(status, ctx=None):
    if status != APT_OK:
        msg = lib().apt_last_error(ctx)
        raise AptError(status, msg.decode() if msg else "")


class Ctx:
    """apt_ctx: rank >= 0 one rank of `world`; rank = -1 emulates all ranks on `device`."""

    def __init__(self, rank=0, world=1, device=0, stream=None):
        self.h = C.c_void_p()
        check(lib().apt_ctx_create(rank, world, device, stream, C.byref(self.h)))
        self.world = world

    def close(self):
        if self.h:
            lib().apt_ctx_destroy(self.h)
            self.h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def ck(self, s):
        check(s, self.h)

    def set_exchange(self, dist, group=None):
        """Multi-process job: install the torch.distributed bootstrap all-gather (collective)."""
        self._xfn = make_exchange(dist, group)
        self.ck(lib().apt_ctx_set_exchange(self.h, self._xfn, None))

    def sync(self):
        self.ck(lib().apt_ctx_sync(self.h))

    def launches(self):
        return lib().apt_ctx_launches(self.h)

    def d2h(self, host: np.ndarray, dev_ptr):
        self.ck(lib().apt_memcpy(self.h, host.ctypes.data, dev_ptr, host.nbytes, 0))
        return host

    # --- objects
    def graph_load(self, indptr, indices, part=None):
        indptr = np.ascontiguousarray(indptr, np.int64)
        indices = np.ascontiguousarray(indices, np.int32)
        part = None if part is None else np.ascontiguousarray(part, np.int32)
        h = C.c_void_p()
        self.ck(lib().apt_graph_load(self.h, len(indptr) - 1, int(indptr[-1]), indptr.ctypes.data,
                                     indices.ctypes.data, _ptr(part), C.byref(h)))
        return Handle(h, lib().apt_graph_destroy, keep=(self,))

    def fstore_create(self, graph, layout, dtype, dim, host_feats=None, feat_seed=0, hbm_frac=1.0, hot_ids=None,
                      counts=None, cache_budget_rows=None):
        """hbm_frac < 1: the rows beyond every shard's HBM budget form the pinned host tier;
        hot_ids: rows replicated into every GPU's spare HBM (excess cache), hottest first.
        counts + cache_budget_rows: P:163's per-strategy GPU caches (APT_CACHE_P163)."""
        h = C.c_void_p()
        hf = None if host_feats is None else np.ascontiguousarray(host_feats, np.float32)
        if counts is not None:
            cnt = np.ascontiguousarray(counts, np.int32)
            o = FstoreOpts(0.0, 0, None, CACHE_P163, cnt.ctypes.data, int(cache_budget_rows))
            self.ck(lib().apt_fstore_create_tiered(self.h, graph.h, layout, dtype, dim, _ptr(hf), feat_seed,
                                                   C.byref(o), C.byref(h)))
            return Handle(h, lib().apt_fstore_destroy, keep=(self, graph, cnt))
        if hbm_frac == 1.0 and hot_ids is None:
            self.ck(lib().apt_fstore_create(self.h, graph.h, layout, dtype, dim, _ptr(hf), feat_seed, C.byref(h)))
            return Handle(h, lib().apt_fstore_destroy, keep=(self, graph))
        hot = None if hot_ids is None else np.ascontiguousarray(hot_ids, np.int64)
        o = FstoreOpts(hbm_frac, 0 if hot is None else len(hot), None if hot is None else hot.ctypes.data)
        self.ck(lib().apt_fstore_create_tiered(self.h, graph.h, layout, dtype, dim, _ptr(hf), feat_seed, C.byref(o),
                                               C.byref(h)))
        return Handle(h, lib().apt_fstore_destroy, keep=(self, graph, hot))

    def sample(self, graph, seeds_dev, n_seeds, fanouts, rng_seed, step):
        f = np.ascontiguousarray(fanouts, np.int32)
        h = C.c_void_p()
        self.ck(lib().apt_sample(self.h, graph.h, _ptr(seeds_dev), n_seeds, f.ctypes.data, len(f), rng_seed, step,
                                 C.byref(h)))
        return Batch(self, h)

    def gather(self, fstore, ids_dev, n, out_dev):
        """apt_gather: ids_dev int64 node ids (ABI rule)."""
        if hasattr(ids_dev, "dtype") and str(ids_dev.dtype) not in ("torch.int64", "int64"):
            raise AptError(1, f"apt_gather: ids must be int64, got {ids_dev.dtype}")
        self.ck(lib().apt_gather(self.h, fstore.h, _ptr(ids_dev), n, _ptr(out_dev)))

    def aggregate(self, view, x_dev, dtype, dim, x_pitch, z_dev, z_pitch):
        self.ck(lib().apt_aggregate(self.h, C.byref(view), _ptr(x_dev), dtype, dim, x_pitch, _ptr(z_dev), z_pitch))

    def aggregate_bwd(self, view, dz_dev, dim, dz_pitch, dx_dev, dx_pitch):
        self.ck(lib().apt_aggregate_bwd(self.h, C.byref(view), _ptr(dz_dev), dim, dz_pitch, _ptr(dx_dev), dx_pitch))

    def project(self, Z_dev, z_pitch, dtype, W_dev, bias_dev, M, N, K, relu, Y_dev, y_pitch):
        self.ck(lib().apt_project(self.h, _ptr(Z_dev), z_pitch, dtype, _ptr(W_dev), _ptr(bias_dev), M, N, K, relu,
                                  _ptr(Y_dev), y_pitch))

    def weight_grad(self, G_dev, g_pitch, Z_dev, z_pitch, dtype, rows, d_out, d_in, dW_dev, db_dev=None):
        self.ck(lib().apt_weight_grad(self.h, _ptr(G_dev), g_pitch, _ptr(Z_dev), z_pitch, dtype, rows, d_out, d_in,
                                      _ptr(dW_dev), _ptr(db_dev)))

    def batch_group(self, batches):
        """apt_batch_group: one batch per hosted rank (emulated ctx) -> a group batch."""
        arr = (C.c_void_p * len(batches))(*[b.h for b in batches])
        h = C.c_void_p()
        self.ck(lib().apt_batch_group(self.h, arr, len(batches), C.byref(h)))
        g = Batch(self, h)
        g._keep = (self,) + tuple(batches)          # the group borrows its members
        return g

    def layer_fwd(self, strategy, batch, fstore, W_dev, bias_dev, d_out, dtype, h1_dev):
        """apt_layer_fwd: the first layer of `batch` under `strategy`; returns
        the saved state for layer_bwd.  h1_dev: fp32 [rows x d_out], ranks concatenated."""
        h = C.c_void_p()
        self.ck(lib().apt_layer_fwd(self.h, strategy, batch.h, fstore.h, _ptr(W_dev), _ptr(bias_dev), d_out, dtype,
                                    _ptr(h1_dev), C.byref(h)))
        return Handle(h, lib().apt_layer_saved_destroy, keep=(self, batch, fstore))

    def layer_bwd(self, saved, dh1_dev, dW_dev, db_dev):
        """apt_layer_bwd: dW [d_out x d] and db [d_out] (device fp32) of the strategy."""
        self.ck(lib().apt_layer_bwd(self.h, saved.h, _ptr(dh1_dev), _ptr(dW_dev), _ptr(db_dev)))

    def profile_links(self):
        bw = BwProfile()
        self.ck(lib().apt_profile_links(self.h, C.byref(bw)))
        return bw


class Handle:
    def __init__(self, h, destroy, keep=()):
        self.h, self._destroy, self._keep = h, destroy, keep

    def close(self):
        if self.h:
            self._destroy(self.h)
            self.h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Batch(Handle):
    def __init__(self, ctx, h):
        super().__init__(h, lib().apt_batch_destroy, keep=(ctx,))
        self.ctx = ctx

    def block(self, hop):
        v = BlockView()
        check(lib().apt_batch_block(self.h, hop, C.byref(v)))
        return v

    def block_host(self, hop):
        """Copy a block to host numpy arrays (dst, src int64 node ids; indptr, indices int32)."""
        v = self.block(hop)
        out = []
        for ptr, n, dt in ((v.dst_ids, v.n_dst, np.int64), (v.src_ids, v.n_src, np.int64),
                           (v.indptr, v.n_dst + 1, np.int32), (v.indices, v.n_edges, np.int32)):
            a = np.empty(n, dt)
            if n:
                self.ctx.d2h(a, ptr)
            out.append(a)
        return out


class Trainer(Handle):
    """apt_trainer: the per-mini-batch step under one strategy."""

    def __init__(self, ctx, graph, fstore, cfg_dims, fanouts, batch, dtype, lr, sample_seed, feat_seed, strategy,
                 labels, gat_heads=0):
        m = ModelDesc()
        m.gat_heads = gat_heads
        m.n_layers = len(fanouts)
        for i, d in enumerate(cfg_dims):
            m.dims[i] = d
        for i, f in enumerate(fanouts):
            m.fanouts[i] = f
        m.batch, m.dtype, m.lr, m.sample_seed, m.feat_seed = batch, dtype, lr, sample_seed, feat_seed
        self._labels = np.ascontiguousarray(labels, np.int32)
        h = C.c_void_p()
        ctx.ck(lib().apt_trainer_create(ctx.h, graph.h, fstore.h, C.byref(m), strategy, self._labels.ctypes.data,
                                        C.byref(h)))
        super().__init__(h, lib().apt_trainer_destroy, keep=(ctx, graph, fstore))
        self.ctx, self.K, self.dims = ctx, len(fanouts), list(cfg_dims)

    def set_params(self, params):
        for l, (W, b) in enumerate(params, start=1):
            W = np.ascontiguousarray(W, np.float32)
            b = np.ascontiguousarray(b, np.float32)
            self.ctx.ck(lib().apt_trainer_set_params(self.h, l, W.ctypes.data, b.ctypes.data))

    def get_params(self, rank=0):
        out = []
        for l in range(1, self.K + 1):
            W = np.empty((self.dims[l], self.dims[l - 1]), np.float32)
            b = np.empty(self.dims[l], np.float32)
            self.ctx.ck(lib().apt_trainer_get_params(self.h, rank, l, W.ctypes.data, b.ctypes.data))
            out.append((W, b))
        return out

    def set_attention(self, a_src, a_dst):
        """GAT layer 1: attention vectors [dims[1]] each (head h at [h*F, (h+1)*F))."""
        a_src = np.ascontiguousarray(a_src, np.float32).reshape(-1)
        a_dst = np.ascontiguousarray(a_dst, np.float32).reshape(-1)
        self.ctx.ck(lib().apt_trainer_set_attention(self.h, a_src.ctypes.data, a_dst.ctypes.data))

    def get_attention(self, rank=0):
        a_src = np.empty(self.dims[1], np.float32)
        a_dst = np.empty(self.dims[1], np.float32)
        self.ctx.ck(lib().apt_trainer_get_attention(self.h, rank, a_src.ctypes.data, a_dst.ctypes.data))
        return a_src, a_dst

    def set_epoch(self, train, epoch):
        train = np.ascontiguousarray(train, np.int64)
        self.ctx.ck(lib().apt_trainer_set_epoch(self.h, train.ctypes.data, len(train), epoch))

    def steps_per_epoch(self):
        return lib().apt_trainer_steps_per_epoch(self.h)

    def step(self, step, update=True):
        self.ctx.ck(lib().apt_trainer_step(self.h, step, 1 if update else 0))

    def step_host(self, gbatch_host, step, update=True):
        loss = C.c_float(0)
        self.ctx.ck(lib().apt_trainer_step_host(self.h, _ptr(gbatch_host), len(gbatch_host), step,
                                                1 if update else 0, C.byref(loss)))
        return loss.value

    def step_host_pipelined(self, next_batch_host, next_step, update=True):
        """Submit the next host batch, run the previously submitted one; returns its loss
        (None for the priming call)."""
        loss, had = C.c_float(0), C.c_int(0)
        self.ctx.ck(lib().apt_trainer_step_host_pipelined(self.h, _ptr(next_batch_host), len(next_batch_host),
                                                          next_step, 1 if update else 0, C.byref(loss),
                                                          C.byref(had)))
        return loss.value if had.value else None

    def step_host_async(self, next_batch_host, next_step, update=True):
        """Submit the next host batch and launch the previously submitted one without waiting
        for it; returns the loss of the step the previous call launched (None at first)."""
        loss, had = C.c_float(0), C.c_int(0)
        self.ctx.ck(lib().apt_trainer_step_host_async(self.h, _ptr(next_batch_host), len(next_batch_host), next_step,
                                                      1 if update else 0, C.byref(loss), C.byref(had)))
        return loss.value if had.value else None

    def loss(self):
        v = C.c_float(0)
        self.ctx.ck(lib().apt_trainer_loss(self.h, C.byref(v)))
        return v.value

    def use_graph(self, on=True):
        self.ctx.ck(lib().apt_trainer_use_graph(self.h, 1 if on else 0))

    def set_pipeline(self, on=True):
        self.ctx.ck(lib().apt_trainer_set_pipeline(self.h, 1 if on else 0))

    def read(self, what, layer=0, rank=0, cap=1 << 28):
        rows, cols = C.c_int64(0), C.c_int(0)
        probe = np.empty(1, np.float32)
        self.ctx.ck(lib().apt_trainer_read(self.h, rank, READ[what], layer, probe.ctypes.data, 0, C.byref(rows),
                                           C.byref(cols)))
        n = rows.value * cols.value
        dt = np.int32 if what in ("seeds", "dst") else np.float32
        out = np.empty(max(n, 1), dt)
        self.ctx.ck(lib().apt_trainer_read(self.h, rank, READ[what], layer, out.ctypes.data, min(n, cap),
                                           C.byref(rows), C.byref(cols)))
        return out[:n].reshape(rows.value, cols.value)

    def phase_ms(self):
        ms = (C.c_double * 6)()
        self.ctx.ck(lib().apt_trainer_phase_ms(self.h, ms, 6))
        return list(ms)

    def layer_fwd(self, step):
        """apt_trainer_layer_fwd: sample step `step` of the epoch, run layer 1."""
        self.ctx.ck(lib().apt_trainer_layer_fwd(self.h, step))

    def layer_bwd(self, dh1_list, pitch):
        """apt_trainer_layer_bwd.  dh1_list: one device tensor per hosted rank (fp32 [rows x pitch])."""
        arr = (C.c_void_p * len(dh1_list))(*[_ptr(x) for x in dh1_list])
        self.ctx.ck(lib().apt_trainer_layer_bwd(self.h, arr, pitch))

    def access_counts(self, n_steps):
        """apt_access_counts: per-node input-row loads over the first n_steps steps (Table 3)."""
        out = np.zeros(len(self._labels), np.int32)   # labels are per node
        self.ctx.ck(lib().apt_access_counts(self.h, n_steps, out.ctypes.data))
        return out

    def dryrun(self, n_steps):
        st = PlanStats()
        self.ctx.ck(lib().apt_dryrun(self.h, n_steps, C.byref(st)))
        return st


def exchange_selftest(rank, world, dist, group=None):
    """Host-only check of the bootstrap all-gather protocol (no GPU)."""
    fn = make_exchange(dist, group)
    check(lib().apt_exchange_selftest(rank, world, fn, None))


PARTITION = {"range": 0, "random": 1, "ldg": 2}


def partition(indptr, indices, n_parts, method="ldg", seed=0):
    """apt_partition: edge-cut partition of a host CSR into n_parts parts (range /
    random / ldg).  Returns (part int32[n], cut_edges)."""
    indptr = np.ascontiguousarray(indptr, np.int64)
    indices = np.ascontiguousarray(indices, np.int32)
    n = len(indptr) - 1
    part = np.empty(n, np.int32)
    cut = C.c_int64(0)
    check(lib().apt_partition(n, int(indptr[-1]), indptr.ctypes.data, indices.ctypes.data, n_parts,
                              PARTITION[method], seed, part.ctypes.data, C.byref(cut)))
    return part, cut.value


CACHE_P163 = 1


def cache_sets(indptr, indices, part, n_parts, strategy, counts, budget):
    """apt_cache_sets: every GPU's cache ids, hottest first."""
    indptr = np.ascontiguousarray(indptr, np.int64)
    indices = np.ascontiguousarray(indices, np.int32)
    part = np.ascontiguousarray(part, np.int32)
    counts = np.ascontiguousarray(counts, np.int32)
    n = len(indptr) - 1
    ids = np.zeros((n_parts, max(budget, 1)), np.int64)
    cnt = np.zeros(n_parts, np.int64)
    check(lib().apt_cache_sets(n, indptr.ctypes.data, indices.ctypes.data, part.ctypes.data, n_parts, strategy,
                               counts.ctypes.data, budget, ids.ctypes.data, cnt.ctypes.data))
    return [ids[r, :cnt[r]].copy() for r in range(n_parts)]


def hot_rows(counts, k):
    """apt_hot_rows: the k most-accessed node ids, descending count, ties by id."""
    counts = np.ascontiguousarray(counts, np.int32)
    out = np.empty(k, np.int64)
    check(lib().apt_hot_rows(counts.ctypes.data, len(counts), k, out.ctypes.data))
    return out


def select_strategy(stats: PlanStats, bw: BwProfile):
    pick = C.c_int(0)
    pred = (C.c_double * 4)()
    check(lib().apt_select_strategy(C.byref(stats), C.byref(bw), C.byref(pick), pred))
    return pick.value, list(pred)
