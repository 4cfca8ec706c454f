"""Multi-GPU drivers (one process per GPU, torch.distributed over NCCL; gloo for the CPU tests).

The labelling pass shards in the two ways SURVEY §8(e) names:

1. Corpus sharding (independent units, "scaling: weak" in bench.py; strong-scaling helper here):
   matrices are assigned to ranks by LPT on an estimated cost, each rank labels its shard with
   ``sfs_label_corpus`` and the fixed-size result rows are gathered once (``all_gather_into_tensor``).
   The paper labels one platform at a time (§5.1); sharding the M×F×N experiments of P:L46
   over GPUs is the build's addition.
2. Row partition of one large matrix (one exchange per SpMV): rank k holds the contiguous row block
   A[r_k:r_{k+1}, :]; each SpMV is either ``all_gather_into_tensor(x_full, x_local)`` followed by the
   local ``sfs_spmv`` (global column ids), or -- SURVEY §8(f) f3 -- a halo exchange: only the ghost
   entries of x the block references, point-to-point from their owners, into an extended vector the
   block's columns were renumbered into (``halo_plan`` / ``rowpart_halo_iterate``).

Everything that touches matrix data runs in libsfs; this module only partitions, launches and
gathers.  The labeller / SpMV callables are injectable so the host logic is testable with gloo on CPU.
"""
from __future__ import annotations

import heapq
from dataclasses import dataclass
from typing import Callable, Dict, List, Optional, Sequence

import numpy as np

# ------------------------------------------------------------------ corpus sharding


def lpt_assign(costs: Sequence[float], world: int) -> List[List[int]]:
    """Longest-processing-time-first: items in decreasing cost (ties by index) each go to the least
    loaded rank (ties to the lowest rank).  Deterministic, identical on every rank; each shard is
    returned in increasing item order."""
    heap = [(0.0, r) for r in range(world)]
    shards: List[List[int]] = [[] for _ in range(world)]
    for i in sorted(range(len(costs)), key=lambda j: (-costs[j], j)):
        load, r = heapq.heappop(heap)
        shards[r].append(i)
        heapq.heappush(heap, (load + float(costs[i]), r))
    return [sorted(s) for s in shards]


def expected_nnz(spec) -> float:
    """Expected nnz of a generator spec (sfsgen classes), from its parameters alone, so that every rank
    can schedule the corpus without generating it.  Scheduling only: nothing here feeds a result.
    band: 1 + 2b·p per row; block-diagonal: 1 + (B−1)·p; uniform: λ (dedup is negligible for n ≫ λ);
    power-law: E[len] = 1 + Σ_{L=2}^{cap} (2/L)^(α−1) (P(len ≥ L) for the inverse-CDF draw, cap =
    min(n, 2^17)); stencils / R-MAT: points per row / edge factor 16."""
    import sfsgen
    m, n = sfsgen.dims(spec)
    c = spec.cls
    if c == sfsgen.BAND:
        per = 1.0 + 2.0 * spec.ia * spec.pa
    elif c == sfsgen.BLOCKDIAG:
        per = 1.0 + (spec.ia - 1) * spec.pa
    elif c == sfsgen.UNIFORM:
        per = spec.pa
    elif c == sfsgen.POWERLAW:
        cap = max(2, min(n, 1 << 17))
        L = np.arange(2, cap + 1, dtype=np.float64)
        per = 1.0 + float(np.sum((2.0 / L) ** (spec.pa - 1.0)))
    elif c == sfsgen.RMAT:
        per = 16.0
    else:
        per = {sfsgen.ST2D5: 5.0, sfsgen.ST3D7: 7.0, sfsgen.ST3D27: 27.0}.get(c, 1.0)
    return float(m) * per


# Race cost model of one matrix (µs): a fixed part (5 formats × 105 dependent launches at the ~3.3 µs
# launch floor, conversions, features) plus a bandwidth part per byte of CSR (all five formats' reps),
# least-squares fit to the corpus-200 race on a B200 (profiles/r01/corpus200_dump.jsonl, r = 0.97).
RACE_FIXED_US = 1740.0
RACE_US_PER_CSR_BYTE = 1.62e-4


def race_cost(spec) -> float:
    return RACE_FIXED_US + RACE_US_PER_CSR_BYTE * (4 + (8 if spec.dtype else 4)) * expected_nnz(spec)


def weak_shard(corpus: int, per_rank: int, rank: int, world: int) -> List[int]:
    """Weak scaling with balanced ranks: the job is the first per_rank·world matrices of the corpus
    recipe, LPT-assigned over the ranks on race_cost, so every rank gets ~per_rank matrices of ~equal
    estimated race time (world = 1: ids [0, per_rank) in order).  Identical on every rank."""
    import sfsgen
    ids = list(range(per_rank * world))
    if world == 1:
        return ids
    costs = [race_cost(sfsgen.corpus_spec(corpus, i)) for i in ids]
    return lpt_assign(costs, world)[rank]


# fixed-size result row gathered across ranks: id, label, matrix status, admissible mask, csr variant,
# t_spmv[5], t_convert[5], status[5], t_features, 23 features  -> 44 float64
RESULT_FIELDS = 44


def pack_result(i: int, feat: dict, lab: dict) -> np.ndarray:
    from . import FEATURE_FLOAT_FIELDS, FEATURE_INT_FIELDS
    row = [i, lab["label"], lab["matrix_status"], lab["admissible_mask"], lab["csr_variant"]]
    row += list(lab["t_spmv_us"]) + list(lab["t_convert_us"]) + list(lab["status"]) + [lab["t_features_us"]]
    row += [feat[k] for k in FEATURE_INT_FIELDS] + [feat[k] for k in FEATURE_FLOAT_FIELDS]
    assert len(row) == RESULT_FIELDS
    return np.array(row, dtype=np.float64)


def unpack_result(row: np.ndarray) -> dict:
    from . import FEATURE_FLOAT_FIELDS, FEATURE_INT_FIELDS
    r = row.tolist()
    out = {"id": int(r[0]), "label": int(r[1]), "matrix_status": int(r[2]), "admissible_mask": int(r[3]),
           "csr_variant": int(r[4]), "t_spmv_us": r[5:10], "t_convert_us": r[10:15],
           "status": [int(v) for v in r[15:20]], "t_features_us": r[20]}
    feats = {}
    for j, k in enumerate(FEATURE_INT_FIELDS):
        feats[k] = int(r[21 + j])
    for j, k in enumerate(FEATURE_FLOAT_FIELDS):
        feats[k] = r[21 + len(FEATURE_INT_FIELDS) + j]
    out["features"] = feats
    return out


def gather_results(local_rows: np.ndarray, world: int, max_per_rank: int, device=None, group=None) -> np.ndarray:
    """all_gather_into_tensor of fixed-size result rows, padded to max_per_rank (pad id = -1).
    Returns every rank's valid rows, sorted by matrix id."""
    import torch
    import torch.distributed as dist
    pad = np.full((max_per_rank, RESULT_FIELDS), -1.0)
    pad[:len(local_rows)] = local_rows
    t = torch.from_numpy(pad.reshape(-1)).to(device or "cpu")
    if world == 1:
        allr = t
    else:
        allr = torch.empty(world * t.numel(), dtype=t.dtype, device=t.device)
        dist.all_gather_into_tensor(allr, t, group=group)
    rows = allr.cpu().numpy().reshape(world * max_per_rank, RESULT_FIELDS)
    rows = rows[rows[:, 0] >= 0]
    return rows[np.argsort(rows[:, 0], kind="stable")]


def label_corpus_sharded(ids: Sequence[int], costs: Sequence[float], make: Callable[[int], object],
                         labeller: Callable[[list], tuple], rank: int, world: int, batch_bytes: float = 40e9,
                         nbytes: Optional[Callable[[object], float]] = None, device=None, group=None) -> List[dict]:
    """Strong-scaling corpus labelling: LPT-shard `ids` (costs aligned), build each matrix with
    `make(id)`, label in memory-bounded batches with `labeller(list_of_matrices) -> (feats, labels)`
    (``sfs.label_corpus`` on a GPU), then gather every rank's results.  Returns the results of ALL
    matrices, in id order, on every rank."""
    shards = lpt_assign(costs, world)
    mine = [ids[j] for j in shards[rank]]
    rows = []
    batch, batch_ids, used = [], [], 0.0
    for i in mine + [None]:
        if i is not None:
            A = make(i)
            b = nbytes(A) if nbytes else 0.0
        if batch and (i is None or used + b > batch_bytes):
            feats, labs = labeller(batch)
            rows += [pack_result(bi, f, L) for bi, f, L in zip(batch_ids, feats, labs)]
            batch, batch_ids, used = [], [], 0.0
        if i is not None:
            batch.append(A)
            batch_ids.append(i)
            used += b
    local = np.stack(rows) if rows else np.zeros((0, RESULT_FIELDS))
    maxn = max(len(s) for s in shards)
    return [unpack_result(r) for r in gather_results(local, world, maxn, device, group)]


# ------------------------------------------------------------------ row partition of one matrix


def row_blocks(m: int, world: int) -> List[int]:
    """Equal contiguous row blocks of ceil(m / world) rows (the last may be short or empty)."""
    b = -(-m // world)
    return [min(m, k * b) for k in range(world + 1)]


def slice_rows(rp: np.ndarray, col: np.ndarray, val: np.ndarray, r0: int, r1: int):
    """Host CSR of rows [r0, r1) with global column ids."""
    a, b = int(rp[r0]), int(rp[r1])
    return (rp[r0:r1 + 1] - a).astype(np.int32), col[a:b].copy(), val[a:b].copy()


@dataclass
class RowPartition:
    m: int
    n: int
    world: int
    rank: int

    @property
    def bounds(self):
        return row_blocks(self.m, self.world)

    @property
    def block(self) -> int:
        return -(-self.m // self.world)

    @property
    def local_rows(self) -> int:
        b = self.bounds
        return b[self.rank + 1] - b[self.rank]


def rowpart_spmv_iterate(part: RowPartition, local_spmv: Callable, x_local, iters: int, group=None,
                         swap: bool = True):
    """`iters` times: x_full = all_gather(x_local) (padded blocks), y_local = A_k x_full[:n]; if swap,
    y_local becomes the next x_local (power-iteration pattern, square A).  Returns y_local.
    `local_spmv(x_full_view, y_local)` runs the rank's SpMV (sfs_spmv on a GPU)."""
    import torch
    import torch.distributed as dist
    blk = part.block
    x_pad = torch.zeros(blk, dtype=x_local.dtype, device=x_local.device)
    x_full = torch.empty(blk * part.world, dtype=x_local.dtype, device=x_local.device)
    y_local = torch.empty(part.local_rows, dtype=x_local.dtype, device=x_local.device)
    cur = x_local
    for _ in range(iters):
        x_pad[:cur.numel()].copy_(cur)
        if part.world > 1:
            dist.all_gather_into_tensor(x_full, x_pad, group=group)
        else:
            x_full.copy_(x_pad)
        local_spmv(x_full[:part.n], y_local)
        if swap:
            cur = y_local.clone()
    return y_local


# ------------------------------------------------------------------ row partition with a halo exchange
# instead of all-gathering all of x before every SpMV (every rank receives (P-1)/P of
# x), each rank receives only the x entries its row block references outside its own slice -- its
# ghost columns -- point-to-point from their owners.  For the 3D 27-point stencil (configs[3]) that is
# two 128^2-row planes per neighbour instead of (P-1)/P of 2^21 rows.  The block's columns are renumbered
# into an extended vector x_ext = [ghosts below r0 | own slice | ghosts at or above r1]; a contiguous
# run of ghosts keeps its offsets, so a banded block stays banded (DIA admissible, same diagonals).
# The SpMV writes y straight into the own-slice view of the next x_ext, the send buffer is packed by
# sfs_gather, and the exchange is one batch of NCCL send/recv pairs.


@dataclass
class HaloPlan:
    world: int
    rank: int
    r0: int
    r1: int
    lo: np.ndarray        # ghost columns < r0, ascending (global ids) -> x_ext[0 : n_lo]
    hi: np.ndarray        # ghost columns >= r1, ascending -> x_ext[n_lo + n_local :]
    recv: List[tuple]     # (source rank, offset in x_ext, count), ascending source
    send: List[tuple]     # (destination rank, offset in the send buffer, count), ascending destination
    send_idx: np.ndarray  # int32 indices into the own slice, concatenated by destination
    col_ext: np.ndarray   # int32 columns of the row block renumbered into x_ext

    @property
    def n_local(self) -> int:
        return self.r1 - self.r0

    @property
    def n_lo(self) -> int:
        return len(self.lo)

    @property
    def n_ext(self) -> int:
        return len(self.lo) + self.n_local + len(self.hi)

    @property
    def recv_count(self) -> int:
        return len(self.lo) + len(self.hi)


def halo_needs(part: RowPartition, col_block: np.ndarray):
    """Ghost columns of a row block: the distinct columns outside the block's own slice [r0, r1)."""
    b = part.bounds
    r0, r1 = b[part.rank], b[part.rank + 1]
    u = np.unique(np.asarray(col_block, dtype=np.int64))
    return u[u < r0], u[u >= r1]


def remap_columns(col_block: np.ndarray, r0: int, r1: int, lo: np.ndarray, hi: np.ndarray) -> np.ndarray:
    c = np.asarray(col_block, dtype=np.int64)
    out = np.empty_like(c)
    below, own, above = c < r0, (c >= r0) & (c < r1), c >= r1
    out[below] = np.searchsorted(lo, c[below])
    out[own] = len(lo) + (c[own] - r0)
    out[above] = len(lo) + (r1 - r0) + np.searchsorted(hi, c[above])
    return out.astype(np.int32)


def _segments(ids: np.ndarray, owner_block: int, base: int):
    """(owner rank, offset, count) runs of an ascending id list, offsets from `base`."""
    segs = []
    if len(ids) == 0:
        return segs
    own = ids // owner_block
    starts = np.flatnonzero(np.r_[True, own[1:] != own[:-1]])
    ends = np.r_[starts[1:], len(ids)]
    for s, e in zip(starts, ends):
        segs.append((int(own[s]), base + int(s), int(e - s)))
    return segs


def build_halo_plan(part: RowPartition, col_block: np.ndarray, requests: Sequence[np.ndarray]) -> HaloPlan:
    """The rank's plan, given `requests[j]` = the global columns rank j needs from this rank (ascending)."""
    b = part.bounds
    r0, r1 = b[part.rank], b[part.rank + 1]
    lo, hi = halo_needs(part, col_block)
    recv = _segments(lo, part.block, 0) + _segments(hi, part.block, len(lo) + (r1 - r0))
    send, idx, off = [], [], 0
    for j, req in enumerate(requests):
        req = np.asarray(req, dtype=np.int64)
        if j == part.rank or len(req) == 0:
            continue
        assert req.min() >= r0 and req.max() < r1, "request outside the owner's slice"
        send.append((j, off, len(req)))
        idx.append(req - r0)
        off += len(req)
    send_idx = (np.concatenate(idx) if idx else np.zeros(0, np.int64)).astype(np.int32)
    return HaloPlan(part.world, part.rank, r0, r1, lo, hi, recv, send, send_idx,
                    remap_columns(col_block, r0, r1, lo, hi))


def halo_requests_by_owner(part: RowPartition, col_block: np.ndarray) -> List[np.ndarray]:
    """What this rank needs from each rank (index j: the columns owned by rank j)."""
    lo, hi = halo_needs(part, col_block)
    g = np.concatenate([lo, hi])
    own = g // part.block
    return [g[own == j] for j in range(part.world)]


def halo_plan(part: RowPartition, col_block: np.ndarray, group=None, device=None) -> HaloPlan:
    """Collective (setup only): every rank tells each owner which of its columns it needs
    (all_to_all_single of the counts, then of the ids), then builds its plan."""
    import torch
    import torch.distributed as dist
    need = halo_requests_by_owner(part, col_block)
    if part.world == 1:
        return build_halo_plan(part, col_block, [np.zeros(0, np.int64)])
    dev = device or "cpu"
    cnt_out = torch.tensor([len(v) for v in need], dtype=torch.int64, device=dev)
    cnt_in = torch.empty(part.world, dtype=torch.int64, device=dev)
    dist.all_to_all_single(cnt_in, cnt_out, group=group)
    cin = cnt_in.cpu().tolist()
    ids_out = torch.from_numpy(np.concatenate(need).astype(np.int64)).to(dev)
    ids_in = torch.empty(int(sum(cin)), dtype=torch.int64, device=dev)
    dist.all_to_all_single(ids_in, ids_out, output_split_sizes=cin, input_split_sizes=[len(v) for v in need],
                           group=group)
    got = ids_in.cpu().numpy()
    req, o = [], 0
    for c in cin:
        req.append(got[o:o + c])
        o += c
    return build_halo_plan(part, col_block, req)


def halo_plans_local(m: int, n: int, world: int, col_blocks: Sequence[np.ndarray]) -> List[HaloPlan]:
    """Every rank's plan built in one process (no collectives): the same plans halo_plan() builds, for
    simulating the P ranks on one GPU and for tests."""
    parts = [RowPartition(m, n, world, k) for k in range(world)]
    needs = [halo_requests_by_owner(parts[k], col_blocks[k]) for k in range(world)]
    return [build_halo_plan(parts[k], col_blocks[k], [needs[j][k] for j in range(world)]) for k in range(world)]


def rowpart_halo_iterate(plan: HaloPlan, local_spmv: Callable, gather: Callable, x_local, iters: int,
                         group=None, ranks: Optional[Sequence[int]] = None):
    """`iters` power-iteration steps y_k = A_k x on the halo plan: exchange ghosts, SpMV into the own
    slice of the other x_ext buffer.  `local_spmv(x_ext, y_view)` runs the rank's remapped block (sfs_spmv
    on a GPU); `gather(x_own_view, idx_tensor, out)` packs the send buffer (sfs_gather).  `ranks`: group
    ranks of the partition's ranks (default: identity).  Returns the final own slice (a view)."""
    import torch
    import torch.distributed as dist
    dev, dt = x_local.device, x_local.dtype
    xa = torch.zeros(plan.n_ext, dtype=dt, device=dev)
    xb = torch.zeros(plan.n_ext, dtype=dt, device=dev)
    own = slice(plan.n_lo, plan.n_lo + plan.n_local)
    xa[own].copy_(x_local)
    idx = torch.from_numpy(plan.send_idx.astype(np.int32)).to(dev)
    sbuf = torch.empty(len(plan.send_idx), dtype=dt, device=dev)
    gr = (lambda k: k) if ranks is None else (lambda k: ranks[k])

    def exchange(buf):
        if plan.world == 1 or (not plan.send and not plan.recv):
            return
        gather(buf[own], idx, sbuf)
        ops = [dist.P2POp(dist.isend, sbuf[o:o + c], gr(j), group=group) for j, o, c in plan.send]
        ops += [dist.P2POp(dist.irecv, buf[o:o + c], gr(j), group=group) for j, o, c in plan.recv]
        for r in dist.batch_isend_irecv(ops):
            r.wait()

    cur, nxt = xa, xb
    exchange(cur)
    for _ in range(iters):
        local_spmv(cur, nxt[own])
        exchange(nxt)
        cur, nxt = nxt, cur
    return cur[own]


# ------------------------------------------------------------------ row partition with the halo push fused in
# SURVEY §8(f) f3, "stores of y into every peer's x": the rank's SpMV kernel itself stores each y entry a
# neighbour needs as a ghost into that neighbour's next x_ext (peer memory: symmetric memory over
# NVLink on one node, or plain device memory when the P ranks are simulated on one GPU), then releases
# a per-(receiver, sender) flag; the neighbour's next SpMV waits on its flags before reading x
# (sfs_spmv_push, include/sfs.h).  No NCCL call and no separate pack / send / unpack per iteration.
# The send entries of a banded / stencil block are contiguous local rows landing in a contiguous run
# of the neighbour's ghost region, so a plan is a handful of runs.


def recv_offsets_by_source(plan: HaloPlan) -> dict:
    """Where each source rank's entries land in this rank's x_ext: {source: offset} (one recv entry per
    source: the ghost ids are sorted and each source owns a contiguous id range, below or above)."""
    out = {}
    for j, o, c in plan.recv:
        assert j not in out, "a source split across the lower and upper ghost regions"
        out[j] = o
    return out


def push_runs(plan: HaloPlan, dst_offset: dict) -> List[tuple]:
    """The rank's pushes as runs (destination rank, local row begin, end, element offset in the
    destination's x_ext).  `dst_offset[j]`: where this rank's entries start in rank j's x_ext (rank j's
    recv_offsets_by_source()[this rank])."""
    runs = []
    for j, o, c in plan.send:
        idx = np.asarray(plan.send_idx[o:o + c], dtype=np.int64)
        if len(idx) == 0:
            continue
        brk = np.flatnonzero(np.diff(idx) != 1) + 1
        starts = np.r_[0, brk]
        ends = np.r_[brk, len(idx)]
        for a, b in zip(starts, ends):
            runs.append((j, int(idx[a]), int(idx[a]) + int(b - a), int(dst_offset[j]) + int(a)))
    return runs


def push_neighbours(plan: HaloPlan) -> List[int]:
    """Ranks this rank waits on and signals: its sources (their ghosts must have arrived) and its
    destinations (they must have finished reading the buffer this rank pushes into)."""
    return sorted({j for j, _, _ in plan.send} | {j for j, _, _ in plan.recv})


def exchange_recv_offsets(plan: HaloPlan, group=None, device=None) -> dict:
    """Collective (setup only): tell every source where its entries land here; returns, for each
    destination of this rank, the offset in the destination's x_ext (push_runs' dst_offset)."""
    import torch
    import torch.distributed as dist
    if plan.world == 1:
        return {}
    dev = device or "cpu"
    mine = recv_offsets_by_source(plan)
    out = torch.tensor([mine.get(j, -1) for j in range(plan.world)], dtype=torch.int64, device=dev)
    inp = torch.empty(plan.world, dtype=torch.int64, device=dev)
    dist.all_to_all_single(inp, out, group=group)
    got = inp.cpu().tolist()
    return {j: int(got[j]) for j, _, _ in plan.send}


def apply_push_host(plans: Sequence[HaloPlan], xs_ext: Sequence[np.ndarray]) -> None:
    """Host model of one push round (tests): every rank's runs copy its own-slice entries into the
    neighbours' x_ext, exactly as the kernels' extra stores do."""
    offs = [recv_offsets_by_source(p) for p in plans]
    for k, p in enumerate(plans):
        dst = {j: offs[j][k] for j, _, _ in p.send}
        for j, b, e, o in push_runs(p, dst):
            xs_ext[j][o:o + (e - b)] = xs_ext[k][p.n_lo + b:p.n_lo + e]


class _PushBuffers:
    """Per-rank device memory of the push protocol: x_ext double buffer, flags[world] (slot per sender),
    counter.  `base(k)` is the address of rank k's block (a peer address in the real multi-GPU case)."""

    def __init__(self, n_ext_max: int, world: int, elem: int):
        self.n_ext_max, self.world, self.elem = n_ext_max, world, elem
        self.x_bytes = n_ext_max * elem
        self.flag_off = 2 * self.x_bytes
        self.counter_off = self.flag_off + 4 * world
        self.nbytes = (self.counter_off + 4 + 255) // 256 * 256

    def x(self, base: int, parity: int) -> int:
        return base + parity * self.x_bytes

    def flag(self, base: int, sender: int) -> int:
        return base + self.flag_off + 4 * sender

    def counter(self, base: int) -> int:
        return base + self.counter_off


def _push_structs(sfs, plan: HaloPlan, runs, nbrs, bases, rank: int, B: _PushBuffers, parity: int, wait: int,
                  sig: int):
    r = [(b, e, B.x(bases[j], parity) + o * B.elem) for j, b, e, o in runs]
    return sfs.push_struct(r, [B.flag(bases[rank], j) for j in nbrs], wait, [B.flag(bases[j], rank) for j in nbrs],
                           sig, B.counter(bases[rank]))


def rowpart_push_iterate_local(plans: Sequence[HaloPlan], mats, fmt: int, x_locals, iters: int, stream=None):
    """The P ranks of a push-fused row partition simulated on ONE GPU (same kernels, same protocol; the
    "peer" buffers are other allocations on this device).  mats[k]: rank k's remapped block converted to
    `fmt` (sfs.Matrix); x_locals[k]: its slice of x.  Each iteration launches every rank's fused SpMV in
    rank order on one stream, so every wait is already satisfied.  Returns the final own slices."""
    import torch
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    world = len(plans)
    dt, dev = x_locals[0].dtype, x_locals[0].device
    B = _PushBuffers(max(p.n_ext for p in plans), world, x_locals[0].element_size())
    mem = [torch.zeros(B.nbytes, dtype=torch.uint8, device=dev) for _ in range(world)]
    bases = [t.data_ptr() for t in mem]
    offs = [recv_offsets_by_source(p) for p in plans]
    runs = [push_runs(p, {j: offs[j][k] for j, _, _ in p.send}) for k, p in enumerate(plans)]
    nbrs = [push_neighbours(p) for p in plans]

    def xview(k, parity):
        n = plans[k].n_ext
        return mem[k][parity * B.x_bytes:parity * B.x_bytes + n * B.elem].view(dt)

    for k, p in enumerate(plans):
        xview(k, 0)[p.n_lo:p.n_lo + p.n_local].copy_(x_locals[k])
    for k, p in enumerate(plans):  # epoch 1: the initial ghosts
        own = xview(k, 0)[p.n_lo:p.n_lo + p.n_local]
        sfs.halo_push(own, _push_structs(sfs, p, runs[k], nbrs[k], bases, k, B, 0, 0, 1), stream)
    for t in range(1, iters + 1):
        cur, nxt = (t - 1) % 2, t % 2
        for k, p in enumerate(plans):
            y = xview(k, nxt)[p.n_lo:p.n_lo + p.n_local]
            sfs.spmv_push(fmt, mats[k], xview(k, cur), y,
                          _push_structs(sfs, p, runs[k], nbrs[k], bases, k, B, nxt, t, t + 1), stream)
    return [xview(k, iters % 2)[p.n_lo:p.n_lo + p.n_local] for k, p in enumerate(plans)], mem


def rowpart_push_iterate(plan: HaloPlan, A_local, fmt: int, x_local, iters: int, group=None, timing=None,
                         transport: str = "ipc"):
    """One rank of the push-fused row partition on a real multi-GPU node: the x_ext double buffer, flags and
    counter live in peer-mapped device memory -- CUDA IPC (`transport="ipc"`: sfs_ipc_alloc / sfs_ipc_open,
    peer access over NVLink; also works for several processes sharing one GPU) or torch symmetric memory
    (`"symm"`, one GPU per rank) -- so the fused kernel's ghost stores go straight into the neighbours'
    HBM.  Setup: one all_to_all of the recv offsets, one all_reduce of the buffer size, an exchange of
    the handles, a barrier.  `timing`: optional dict receiving the per-iteration device time (ms)."""
    import torch
    import torch.distributed as dist
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    dev, dt = x_local.device, x_local.dtype
    multi = plan.world > 1
    nmax = torch.tensor([plan.n_ext], dtype=torch.int64, device=dev if dist.is_initialized() and
                        dist.get_backend(group) == "nccl" else "cpu")
    if multi:
        dist.all_reduce(nmax, op=dist.ReduceOp.MAX, group=group)
    B = _PushBuffers(int(nmax.item()), plan.world, x_local.element_size())
    opened, own_ipc, keep = [], None, None
    if multi and transport == "symm":
        import torch.distributed._symmetric_memory as symm_mem
        keep = symm_mem.empty(B.nbytes, dtype=torch.uint8, device=dev)
        keep.zero_()
        hdl = symm_mem.rendezvous(keep, group if group is not None else dist.group.WORLD)
        bases = [int(p) for p in hdl.buffer_ptrs]
    elif multi:
        own_ipc, h = sfs.ipc_alloc(B.nbytes)
        handles = [None] * plan.world
        dist.all_gather_object(handles, h, group=group)
        bases = []
        for j, hj in enumerate(handles):
            if j == plan.rank:
                bases.append(own_ipc)
            else:
                bases.append(sfs.ipc_open(hj))
                opened.append(bases[-1])
    else:  # no neighbours: the fused kernel's protocol runs on local memory only
        keep = torch.zeros(B.nbytes, dtype=torch.uint8, device=dev)
        bases = [keep.data_ptr()]
    own_base = bases[plan.rank]
    raw = keep if keep is not None else _device_bytes(own_base, B.nbytes, dev)
    runs = push_runs(plan, exchange_recv_offsets(plan, group, nmax.device))
    nbrs = push_neighbours(plan)
    k = plan.rank
    xv = lambda parity: raw[parity * B.x_bytes:parity * B.x_bytes + plan.n_ext * B.elem].view(dt)
    own = slice(plan.n_lo, plan.n_lo + plan.n_local)
    xv(0)[own].copy_(x_local)
    torch.cuda.synchronize()
    if multi:
        dist.barrier(group=group)
    sfs.halo_push(xv(0)[own], _push_structs(sfs, plan, runs, nbrs, bases, k, B, 0, 0, 1))
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for t in range(1, iters + 1):
        cur, nxt = (t - 1) % 2, t % 2
        sfs.spmv_push(fmt, A_local, xv(cur), xv(nxt)[own],
                      _push_structs(sfs, plan, runs, nbrs, bases, k, B, nxt, t, t + 1))
    e1.record()
    torch.cuda.synchronize()
    if timing is not None:
        timing["ms_per_iter"] = e0.elapsed_time(e1) / max(iters, 1)
    out = xv(iters % 2)[own].clone()
    torch.cuda.synchronize()
    if multi:
        dist.barrier(group=group)  # every neighbour is done storing into our buffer
    for a in opened:
        sfs.ipc_close(a)
    if multi:
        dist.barrier(group=group)
    if own_ipc is not None:
        sfs.ipc_free(own_ipc)
    return out


def _device_bytes(addr: int, nbytes: int, dev):
    """A uint8 torch view of library-allocated device memory (no copy, not owned by torch)."""
    import torch

    class _Mem:
        __cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (addr, False), "version": 3}

    return torch.as_tensor(_Mem(), device=dev)
