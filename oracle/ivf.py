"""Oracle for batched IVF k-NN (§3.1, §3.3, §4.1 strategy B).  TEST INFRASTRUCTURE ONLY.

Notation follows the paper: m queries q_1..q_m, n data vectors v_1..v_n, top-k per query
(§3.2.1); a coarse codebook C of nlist centroids with I(v) = the closest
centroid (§3.1); nprobe closest buckets per query, then a scan of those
buckets with the fine quantizer (§3.1).

Everything is float64 (inputs are fp32 arrays, widened), except the SQ8 codec which the
index stores in fp32 (reading O3).  No blocking, fusion or reordering beyond
the definitions: distances are computed per (query, candidate) pair, orders come from a
full lexicographic sort.
"""
from __future__ import annotations

import numpy as np

L2 = 0  # squared Euclidean distance, smaller is better          (§2.1)
IP = 1  # inner product, larger is better                         (§2.1)
FLAT = 0  # IVF_FLAT: original vectors                            (§3.1)
SQ8 = 1  # IVF_SQ8: one byte per dimension                        (§3.1)

PAD_ID = -1


def pad_value(metric: int) -> float:
    """Distance reported for padding slots (fewer than k candidates): the worst value."""
    return np.inf if metric == L2 else -np.inf


# ----------------------------------------------------------------------------------------
# distances (§2.1: Euclidean and inner product)
# ----------------------------------------------------------------------------------------
def distances(q: np.ndarray, X: np.ndarray, metric: int) -> np.ndarray:
    """D[i] between one query q (d,) and each row of X (n, d), float64.

    L2 is the SQUARED Euclidean distance sum_j (q_j - x_j)^2 (reading O1: squaring is
    monotone, so the ranking is the paper's Euclidean ranking).  IP is sum_j q_j x_j."""
    q = np.asarray(q, dtype=np.float64)
    X = np.asarray(X, dtype=np.float64)
    if metric == L2:
        diff = X - q[None, :]
        return (diff * diff).sum(axis=1)
    return (X * q[None, :]).sum(axis=1)


def _order(D: np.ndarray, ids: np.ndarray, rows: np.ndarray, metric: int) -> np.ndarray:
    """Best-first total order: by distance (ascending L2 / descending IP), then smaller id,
    then storage row (reading O1: the paper records ids tied at d_l, §3.3,
    but does not fix an order among ties)."""
    primary = D if metric == L2 else -D
    return np.lexsort((rows, ids, primary))


def select_topk(D, ids, rows, k: int, metric: int):
    """Plain definition of top-k: sort all candidates by the total order, take the first k,
    pad with (PAD_ID, worst) when fewer than k exist.  Returns (dist[k], id[k], row[k])."""
    D = np.asarray(D, dtype=np.float64)
    ids = np.asarray(ids, dtype=np.int64)
    rows = np.asarray(rows, dtype=np.int64)
    o = _order(D, ids, rows, metric)[:k]
    outD = np.full(k, pad_value(metric), dtype=np.float64)
    outI = np.full(k, PAD_ID, dtype=np.int64)
    outR = np.full(k, -1, dtype=np.int64)
    outD[: len(o)] = D[o]
    outI[: len(o)] = ids[o]
    outR[: len(o)] = rows[o]
    return outD, outI, outR


def bit_is_set(bitset, nbits: int, ids: np.ndarray) -> np.ndarray:
    """Exclusion bitset of strategy B (§4.1): a bitmap of entity ids tested
    "whenever a vector is encountered".  Reading: bit = 1 means EXCLUDED
    (deleted / failing the attribute constraint); bit i is byte i>>3, position i&7; ids >= nbits
    (and negative ids) are never excluded."""
    ids = np.asarray(ids, dtype=np.int64)
    out = np.zeros(ids.shape, dtype=bool)
    if bitset is None or nbits <= 0:
        return out
    b = np.asarray(bitset, dtype=np.uint8)
    inside = (ids >= 0) & (ids < nbits)
    ii = ids[inside]
    out[inside] = ((b[ii >> 3] >> (ii & 7)) & 1).astype(bool)
    return out


# ----------------------------------------------------------------------------------------
# exact k-NN (the problem statement, §3.2.1; ground truth)
# ----------------------------------------------------------------------------------------
def exact_knn(X, ids, Q, k: int, metric: int, bitset=None, nbits: int = 0):
    """Brute force: every query against every non-excluded vector, full sort, first k.
    Rows are the positions in X.  Returns (D[m,k] float64, I[m,k] int64)."""
    X = np.asarray(X)
    ids = np.asarray(ids, dtype=np.int64)
    Q = np.asarray(Q)
    keep = ~bit_is_set(bitset, nbits, ids)
    rows = np.nonzero(keep)[0]
    m = Q.shape[0]
    outD = np.empty((m, k), dtype=np.float64)
    outI = np.empty((m, k), dtype=np.int64)
    for i in range(m):
        D = distances(Q[i], X[rows], metric)
        outD[i], outI[i], _ = select_topk(D, ids[rows], rows, k, metric)
    return outD, outI


# ----------------------------------------------------------------------------------------
# coarse quantizer (§3.1)
# ----------------------------------------------------------------------------------------
def assign(X, C, metric: int) -> np.ndarray:
    """I(v) = the closest centroid.  L2: argmin ||v - c||^2; IP: argmax <v, c>
    (reading O2: "closest" under the index metric).  Ties -> smaller centroid id (np.argmin /
    np.argmax return the first extremum)."""
    X = np.asarray(X)
    out = np.empty(X.shape[0], dtype=np.int64)
    for i in range(X.shape[0]):
        s = distances(X[i], C, metric)
        out[i] = np.argmin(s) if metric == L2 else np.argmax(s)
    return out


def probe(Q, C, nprobe: int, metric: int) -> np.ndarray:
    """Step (1) of IVF query processing: "find the closest nprobe buckets ... based on the
    distance between q and the centroid of each bucket" (§3.1).  Per query
    the first nprobe centroids by (distance best-first, centroid id); nprobe > nlist is clamped.
    Returns P[m, nprobe'] int64, best-first."""
    C = np.asarray(C)
    nlist = C.shape[0]
    npb = min(nprobe, nlist)
    Q = np.asarray(Q)
    P = np.empty((Q.shape[0], npb), dtype=np.int64)
    lid = np.arange(nlist, dtype=np.int64)
    for i in range(Q.shape[0]):
        s = distances(Q[i], C, metric)
        P[i] = _order(s, lid, lid, metric)[:npb]
    return P


# ----------------------------------------------------------------------------------------
# SQ8 scalar quantizer (§3.1: "compress a 4-byte float value to a 1-byte
# integer"; PAPER.md:803 fn. 6: 1/4 the space of IVF_FLAT).  The paper gives no formula:
# reading O3 = per-dimension min/max range, truncating encode, mid-bin decode,
# no residual, all in fp32 with one rounding per operation.
# ----------------------------------------------------------------------------------------
def sq8_train(sample):
    """vmin_j = min over the sample, vdiff_j = max_j - min_j (fp32)."""
    S = np.asarray(sample, dtype=np.float32)
    vmin = S.min(axis=0).astype(np.float32)
    vmax = S.max(axis=0).astype(np.float32)
    vdiff = (vmax - vmin).astype(np.float32)
    return vmin, vdiff


def sq8_encode(X, vmin, vdiff) -> np.ndarray:
    """code = floor(255 * clamp((x - vmin)/vdiff, 0, 1)) with t = 0 where vdiff = 0.
    fp32, each operation rounded to nearest (numpy float32 elementwise ops, no FMA)."""
    X = np.asarray(X, dtype=np.float32)
    vmin = np.asarray(vmin, dtype=np.float32)
    vdiff = np.asarray(vdiff, dtype=np.float32)
    num = (X - vmin[None, :]).astype(np.float32)
    safe = np.where(vdiff > 0, vdiff, np.float32(1)).astype(np.float32)
    t = (num / safe[None, :]).astype(np.float32)
    t = np.where(vdiff[None, :] > 0, t, np.float32(0))
    t = np.clip(t, np.float32(0), np.float32(1)).astype(np.float32)
    code = np.floor((np.float32(255) * t).astype(np.float32))
    return code.astype(np.uint8)


def sq8_decode(codes, vmin, vdiff) -> np.ndarray:
    """x_hat = vmin + ((code + 0.5) / 255) * vdiff, fp32, evaluated in that order."""
    c = np.asarray(codes, dtype=np.float32)
    vmin = np.asarray(vmin, dtype=np.float32)
    vdiff = np.asarray(vdiff, dtype=np.float32)
    t = ((c + np.float32(0.5)).astype(np.float32) / np.float32(255)).astype(np.float32)
    return (t * vdiff[None, :]).astype(np.float32) + vmin[None, :]


# ----------------------------------------------------------------------------------------
# the IVF index (§3.1)
# ----------------------------------------------------------------------------------------
class IvfIndex:
    """Buckets = the vectors whose closest centroid is c.  Storage is
    list-major: bucket 0's vectors in insertion order, then bucket 1's, ...; a vector's
    storage row is its position there (used only to order exact (dist, id) ties)."""

    def __init__(self, d: int, metric: int, kind: int, centroids):
        self.d, self.metric, self.kind = d, metric, kind
        self.C = np.asarray(centroids, dtype=np.float32).reshape(-1, d)
        self.nlist = self.C.shape[0]
        self.vmin = self.vdiff = None
        self._vecs = np.zeros((0, d), dtype=np.float32)    # raw added vectors, insertion order
        self._ids = np.zeros(0, dtype=np.int64)
        self._list = np.zeros(0, dtype=np.int64)

    def set_sq8(self, vmin, vdiff):
        self.vmin = np.asarray(vmin, dtype=np.float32)
        self.vdiff = np.asarray(vdiff, dtype=np.float32)

    def train_sq8(self, sample):
        self.set_sq8(*sq8_train(sample))

    def add(self, X, ids, lists=None):
        """Insert: assign each vector to I(v) (or take `lists` -- the conditional-oracle
        protocol re-runs the scan with another implementation's accepted assignment)."""
        X = np.asarray(X, dtype=np.float32).reshape(-1, self.d)
        ids = np.asarray(ids, dtype=np.int64)
        a = assign(X, self.C, self.metric) if lists is None else np.asarray(lists, dtype=np.int64)
        self._vecs = np.concatenate([self._vecs, X])
        self._ids = np.concatenate([self._ids, ids])
        self._list = np.concatenate([self._list, a])

    @property
    def ntotal(self) -> int:
        return len(self._ids)

    def storage(self):
        """(list_off[nlist+1], order) with order = insertion indices in list-major order."""
        order = np.lexsort((np.arange(self.ntotal), self._list))
        counts = np.bincount(self._list, minlength=self.nlist)
        off = np.zeros(self.nlist + 1, dtype=np.int64)
        off[1:] = np.cumsum(counts)
        return off, order

    def stored_vectors(self, order) -> np.ndarray:
        """What the fine quantizer keeps: FLAT = the vectors; SQ8 = their decoded codes."""
        V = self._vecs[order]
        if self.kind == SQ8:
            return sq8_decode(sq8_encode(V, self.vmin, self.vdiff), self.vmin, self.vdiff)
        return V

    def codes(self, order) -> np.ndarray:
        return sq8_encode(self._vecs[order], self.vmin, self.vdiff)

    def search(self, Q, k: int, nprobe: int, bitset=None, nbits: int = 0, probes=None):
        """Two-step IVF query processing (§3.1) with strategy B's bitmap
        checked for every encountered vector before the top-k (§4.1).
        Step 1: P = probe(...) (or the given `probes`).  Step 2: candidates = members of the
        probed buckets not excluded; distance to the stored (FLAT) or decoded (SQ8) vector;
        exact top-k by the total order.  Returns (D[m,k] float64, I[m,k] int64, R[m,k] rows)."""
        Q = np.asarray(Q, dtype=np.float32).reshape(-1, self.d)
        P = probe(Q, self.C, nprobe, self.metric) if probes is None else np.asarray(probes)
        off, order = self.storage()
        V = self.stored_vectors(order)
        ids = self._ids[order]
        excl = bit_is_set(bitset, nbits, ids)
        m = Q.shape[0]
        outD = np.empty((m, k), dtype=np.float64)
        outI = np.empty((m, k), dtype=np.int64)
        outR = np.empty((m, k), dtype=np.int64)
        for i in range(m):
            rows = np.concatenate([np.arange(off[l], off[l + 1]) for l in P[i]] + [np.zeros(0, np.int64)])
            rows = rows[~excl[rows]]
            D = distances(Q[i], V[rows], self.metric)
            outD[i], outI[i], outR[i] = select_topk(D, ids[rows], rows, k, self.metric)
        return outD, outI, outR


# ----------------------------------------------------------------------------------------
# large k by rounds (§3.3) -- cross-check of the plain definition only
# ----------------------------------------------------------------------------------------
def topk_rounds(D, ids, rows, k: int, metric: int, round_k: int = 1024):
    """The paper's multi-round top-k for k > 1024: round 1 takes the best `round_k`; each
    later round looks at d_l (the last result of the previous round), filters out vectors
    better than d_l and those tied at d_l that were already recorded, takes the next
    `round_k` from the rest and appends them; stop when k results are collected.  Ties are
    recorded by (id, row) so that duplicate ids cannot be lost (reading)."""
    D = np.asarray(D, dtype=np.float64)
    ids = np.asarray(ids, dtype=np.int64)
    rows = np.asarray(rows, dtype=np.int64)
    key = D if metric == L2 else -D
    taken_D, taken_I, taken_R = [], [], []
    alive = np.ones(len(D), dtype=bool)
    while len(taken_D) < k and alive.any():
        idx = np.nonzero(alive)[0]
        o = idx[_order(D[idx], ids[idx], rows[idx], metric)[:round_k]]
        taken_D += list(D[o]); taken_I += list(ids[o]); taken_R += list(rows[o])
        d_l = key[o[-1]]
        recorded = set(zip(ids[o][key[o] == d_l].tolist(), rows[o][key[o] == d_l].tolist()))
        tie_rec = np.array([(i, r) in recorded for i, r in zip(ids.tolist(), rows.tolist())], dtype=bool)
        alive &= ~(key < d_l) & ~tie_rec
    outD = np.full(k, pad_value(metric)); outI = np.full(k, PAD_ID, dtype=np.int64)
    n = min(k, len(taken_D))
    outD[:n] = taken_D[:n]; outI[:n] = taken_I[:n]
    return outD, outI


# ----------------------------------------------------------------------------------------
# merging per-segment results (§3.2.1 heap merge; 773-776 §3.3 segments)
# ----------------------------------------------------------------------------------------
def merge_topk(parts, k: int, metric: int):
    """Top-k of the union of per-shard top-k lists [(D[m,k_s], I[m,k_s]), ...] under the total
    order (distance, id, shard, position); padding entries (id -1) are dropped."""
    m = parts[0][0].shape[0]
    outD = np.empty((m, k)); outI = np.empty((m, k), dtype=np.int64)
    for i in range(m):
        Ds, Is, Rs = [], [], []
        for s, (D, I) in enumerate(parts):
            keep = np.asarray(I[i]) != PAD_ID
            Ds.append(np.asarray(D[i], dtype=np.float64)[keep]); Is.append(np.asarray(I[i])[keep])
            Rs.append(s * (1 << 32) + np.nonzero(keep)[0])
        outD[i], outI[i], _ = select_topk(np.concatenate(Ds), np.concatenate(Is), np.concatenate(Rs), k, metric)
    return outD, outI


# ----------------------------------------------------------------------------------------
# recall (§7.1): |S ∩ S'| / |S|
# ----------------------------------------------------------------------------------------
def recall_at_k(I_true, I_ret, k: int) -> float:
    I_true = np.asarray(I_true)[:, :k]
    I_ret = np.asarray(I_ret)[:, :k]
    hit = tot = 0
    for t, r in zip(I_true, I_ret):
        S = set(t[t != PAD_ID].tolist())
        Sp = set(r[r != PAD_ID].tolist())
        hit += len(S & Sp)
        tot += len(S)
    return hit / max(tot, 1)
