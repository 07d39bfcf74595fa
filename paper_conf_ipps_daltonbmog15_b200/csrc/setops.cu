// setops.cu -- balanced-path set operations on sorted key lists (sm_100a).
//
// Paper: Section III-B, the paper's second contribution
// and its Fig 2 benchmark: union, intersection, difference and symmetric
// difference of two sorted lists with duplicates, keys only or key-value
// pairs, 32- or 64-bit.  Duplicates are key-rank pairs: the r-th copy of a key
// in A matches the r-th copy in B, so items are ordered by
// (key, rank, A first) and balanced path keeps every matched pair on one side
// of every cut -- reading R4; for unique keys it is the Z23 shift.
//
// B200 design: ONE pass over the data.
//   * partition kernel: one thread per tile boundary, merge-path search over
//     A and B in global memory, then the balanced-path fix-up inside the run
//     of equal keys the cut falls in;
//   * tile kernel (one CTA per tile of T items, tiles claimed in order by an
//     atomic ticket): coalesced staging of the tile's A and B windows (keys
//     and values) in shared memory, per-thread balanced-path split in shared
//     memory, serial walk counting the outputs, CTA scan, decoupled look-back
//     over the tiles for the global output offset, second walk writing the
//     outputs.  The result size comes back with the last tile's prefix.
#include <algorithm>
#include <climits>
#include <cstdint>

#include "common.cuh"
#include "internal.h"

namespace msp {
namespace {

#ifndef MSP_SET_NT
#define MSP_SET_NT 256
#endif
constexpr int SET_NT = MSP_SET_NT;
#ifndef MSP_SET_IPT
#define MSP_SET_IPT 12
#endif
constexpr int SET_IPT = MSP_SET_IPT;
#ifndef MSP_SET_MINB
#define MSP_SET_MINB 1
#endif
constexpr int SET_T = SET_NT * SET_IPT;  // merge items per tile (+1 for a starred cut)
constexpr int SET_STEPS = SET_IPT + 1;  // register output slots per thread

struct Cut {
    int64_t i, j;
};

template <typename KT, typename IT, class LA, class LB>
__device__ __forceinline__ Cut balanced_fixup(LA A, IT na, LB B, IT nb, const IT i, const IT j);

// Balanced-path cut of diagonal d over key arrays A[0..na), B[0..nb)
// (global or shared memory, any key type; IT = index type, int64_t in global
// memory, int inside a tile).  See partition_model.py
// balanced_path_split_ranked for the reference statement of the rule.
template <typename KT, typename IT, class LA, class LB>
__device__ __forceinline__ Cut balanced_cut(LA A, IT na, LB B, IT nb, IT d)
{
    IT lo = d > nb ? d - nb : 0, hi = d < na ? d : na;
    while (lo < hi) {  // merge path, A first on ties (Alg. 1)
        const IT mid = (lo + hi) >> 1;
        if (A(mid) <= B(d - mid - 1)) lo = mid + 1;
        else hi = mid;
    }
    return balanced_fixup<KT, IT>(A, na, B, nb, lo, d - lo);
}

// The balanced-path fix-up of a merge-path cut (i, j): if the
// cut falls inside a run of equal keys, move it to the ranked position.
template <typename KT, typename IT, class LA, class LB>
__device__ __forceinline__ Cut balanced_fixup(LA A, IT na, LB B, IT nb, const IT i, const IT j)
{
    const bool hl = i > 0 || j > 0, hn = i < na || j < nb;
    if (!hl || !hn) return Cut{i, j};
    KT last = 0, next = ~KT(0);
    if (i > 0) last = A(i - 1);
    if (j > 0 && B(j - 1) > last) last = B(j - 1);
    if (i < na) next = A(i);
    if (j < nb && B(j) < next) next = B(j);
    if (last != next) return Cut{i, j};  // the cut is between two keys
    const KT k = last;
    // bounds of the run of key k around position x: galloping from x (runs
    // are short next to the arrays), then bisection inside the bracket
    auto lower = [&](auto X, IT x) {  // first index in [0, x] with X >= k (X(x) >= k or x == end)
        IT step = 1, h = x;
        while (h > 0 && X(h - 1) == k) {
            const IT l = h > step ? h - step : 0;
            if (X(l) < k) {
                IT a = l + 1, b = h - 1;  // X(l) < k, X(b) == k: first >= k in (l, b]
                while (a < b) {
                    const IT m = (a + b) >> 1;
                    if (X(m) < k) a = m + 1;
                    else b = m;
                }
                return a;
            }
            h = l;
            step <<= 1;
        }
        return h;
    };
    auto upper = [&](auto X, IT x, IT n) {  // first index in [x, n] with X > k
        IT step = 1, l = x;
        while (l < n && X(l) == k) {
            const IT h = n - l > step ? l + step : n;
            if (h == n || X(h) > k) {
                IT a = l + 1, b = h;  // X(l) == k, X(h) > k (or h == n): first > k in (l, h]
                while (a < b) {
                    const IT m = (a + b) >> 1;
                    if (X(m) <= k) a = m + 1;
                    else b = m;
                }
                return a;
            }
            l = h;  // X(h) == k
            step <<= 1;
        }
        return l;
    };
    const IT a_lo = lower(A, i), a_hi = upper(A, i, na);
    const IT b_lo = lower(B, j), b_hi = upper(B, j, nb);
    const IT ca = a_hi - a_lo, cb = b_hi - b_lo;
    const IT p = (i - a_lo) + (j - b_lo);  // items of key k before the cut
    const IT mm = ca < cb ? ca : cb;
    IT ia, ib;
    if (p <= 2 * mm) {
        ia = (p + 1) >> 1;
        ib = p >> 1;
        if (ia > ib) ++ib;  // starred: the matched B copy joins the left side
    } else if (ca > cb) {
        ia = p - cb;
        ib = cb;
    } else {
        ia = ca;
        ib = p - ca;
    }
    return Cut{a_lo + ia, b_lo + ib};
}

// One thread per tile boundary.  (A warp per boundary doing a 32-ary search
// was measured slower on B200: 80 us vs 31 us at 1e8 keys, its 64 random
// probes per round cost more DRAM sectors than the binary search's latency.)
template <typename KT>
__global__ void set_partition_kernel(const KT *__restrict__ A, int64_t na, const KT *__restrict__ B, int64_t nb,
                                     int64_t ntiles, Cut *__restrict__ cuts, uint64_t *__restrict__ states,
                                     unsigned *__restrict__ ticket, int64_t *__restrict__ nC)
{
    const int64_t total = na + nb;
    // also clears the tile kernel's look-back state, ticket and result words
    // (one launch fewer than a separate memset; the tile kernel runs after
    // this one on the same stream)
    if (blockIdx.x == 0 && threadIdx.x < 4) ticket[threadIdx.x] = 0u;
    if (blockIdx.x == 0 && threadIdx.x < 2) nC[threadIdx.x] = 0;
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k <= ntiles;
         k += int64_t(gridDim.x) * blockDim.x) {
        if (k < ntiles) states[k] = 0ull;
        const int64_t d = k * SET_T < total ? k * SET_T : total;
        cuts[k] = balanced_cut<KT, int64_t>([&](int64_t x) { return A[x]; }, na, [&](int64_t x) { return B[x]; }, nb, d);
    }
}

template <int VB> struct ValT { using T = uint32_t; };
template <> struct ValT<8> { using T = uint64_t; };

template <typename KT, int VB>
struct SetSmem {
    KT ka[SET_T + 2];
    KT kb[SET_T + 2];
    typename ValT<VB>::T va[VB ? SET_T + 2 : 1];
    typename ValT<VB>::T vb[VB ? SET_T + 2 : 1];
    int cut_i[SET_NT + 1], cut_j[SET_NT + 1];
    int wsum[SET_NT / 32];
    int64_t base;
    int tile;
};

constexpr uint64_t ST_AGG = 1ull << 62, ST_PRE = 2ull << 62, ST_VAL = (1ull << 62) - 1;

// op: 0 union, 1 intersection, 2 difference (A - B), 3 symmetric difference
template <typename KT, int VB, int OP>
__global__ void __launch_bounds__(SET_NT, MSP_SET_MINB)
set_tile_kernel(const KT *__restrict__ A, const void *__restrict__ Av, int64_t na, const KT *__restrict__ B,
                const void *__restrict__ Bv, int64_t nb, const Cut *__restrict__ cuts, int64_t ntiles,
                uint64_t *__restrict__ states, unsigned *__restrict__ ticket, KT *__restrict__ C,
                void *__restrict__ Cv, int64_t cap, int64_t *__restrict__ nC, unsigned *__restrict__ bad)
{
    using VT = typename ValT<VB>::T;
    constexpr bool EA = (OP == 0 || OP == 2 || OP == 3), EB = (OP == 0 || OP == 3), EM = (OP == 0 || OP == 1);
    extern __shared__ __align__(16) char smem_raw[];
    SetSmem<KT, VB> &S = *reinterpret_cast<SetSmem<KT, VB> *>(smem_raw);
    const int tid = threadIdx.x;
#ifdef MSP_SET_BLOCKID_TILES  // experiment: tile = blockIdx.x (relies on in-order CTA dispatch)
    const int tile = int(blockIdx.x);
#else
    if (tid == 0) S.tile = int(atomicAdd(ticket, 1u));  // tiles in claim order: look-back never waits on an unstarted tile
    __syncthreads();
    const int tile = S.tile;
#endif
    const Cut c0 = cuts[tile], c1 = cuts[tile + 1];
    // Unsorted input (a contract violation) can give non-monotone or oversized
    // cuts: flag it (the call returns MSP_ERR_INPUT) and clamp the windows so
    // every shared-memory and global access stays in bounds.
    const int64_t la64 = c1.i - c0.i, lb64 = c1.j - c0.j;
    const bool bad_cut = la64 < 0 || lb64 < 0 || la64 + lb64 > SET_T + 1;
    const int la = int(la64 < 0 ? 0 : la64 > SET_T + 1 ? SET_T + 1 : la64);
    const int lb = int(lb64 < 0 ? 0 : lb64 > SET_T + 1 ? SET_T + 1 : lb64);
    if (tid == 0 && bad_cut) atomicOr(bad, 1u);
    // stage both windows with asynchronous element copies (LDGSTS): every
    // copy of the tile is in flight at once, no register round trip
    for (int x = tid; x < la; x += SET_NT) {
        cp_async<sizeof(KT)>(&S.ka[x], &A[c0.i + x]);
        if constexpr (VB > 0) cp_async<VB>(&S.va[x], static_cast<const VT *>(Av) + c0.i + x);
    }
    for (int x = tid; x < lb; x += SET_NT) {
        cp_async<sizeof(KT)>(&S.kb[x], &B[c0.j + x]);
        if constexpr (VB > 0) cp_async<VB>(&S.vb[x], static_cast<const VT *>(Bv) + c0.j + x);
    }
    cp_async_wait_all();
    __syncthreads();
    {  // contract check: keys ascending inside the windows and across the
       // window edges (with monotone cuts the windows tile A and B exactly)
        bool uns = false;
        for (int x = tid; x + 1 < la; x += SET_NT) uns |= S.ka[x + 1] < S.ka[x];
        for (int x = tid; x + 1 < lb; x += SET_NT) uns |= S.kb[x + 1] < S.kb[x];
        if (tid == 0 && la > 0 && c0.i > 0 && c0.i < na) uns |= S.ka[0] < A[c0.i - 1];
        if (tid == 1 && lb > 0 && c0.j > 0 && c0.j < nb) uns |= S.kb[0] < B[c0.j - 1];
        if (uns) atomicOr(bad, 1u);
    }
    {  // this thread's cut inside the tile (windows clipped to the tile: consistent, R4)
        const int d = min(tid * SET_IPT, la + lb);
        const Cut c = balanced_cut<KT, int>([&](int x) { return S.ka[x]; }, la, [&](int x) { return S.kb[x]; }, lb, d);
        S.cut_i[tid] = int(c.i);
        S.cut_j[tid] = int(c.j);
        if (tid == 0) {
            S.cut_i[SET_NT] = la;
            S.cut_j[SET_NT] = lb;
        }
    }
    __syncthreads();
    // a starred cut may pass the next thread's nominal diagonal: clamp (monotone)
    int ia0 = S.cut_i[tid], ib0 = S.cut_j[tid];
    int ia1 = max(S.cut_i[tid + 1], ia0), ib1 = max(S.cut_j[tid + 1], ib0);
    // A thread's window holds <= SET_IPT + 1 items (its end cut may be starred)
    // and every walk step consumes >= 1 of them, so SET_STEPS register slots
    // hold its outputs; a CTA where that fails takes the two-walk path.
#ifdef MSP_SET_FORCE_WALK2  // test build: exercise the two-walk path
    const bool regs = __syncthreads_and(ia1 < ia0);
#else
    const bool regs = __syncthreads_and((ia1 - ia0) + (ib1 - ib0) <= SET_STEPS);
#endif
    auto walk = [&](auto &&emit) {
        int ia = ia0, ib = ib0;
        while (ia < ia1 || ib < ib1) {
            const bool ra = ia < ia1, rb = ib < ib1;
            if (ra && (!rb || S.ka[ia] < S.kb[ib])) {
                if (EA) emit(true, ia);
                ++ia;
            } else if (rb && (!ra || S.kb[ib] < S.ka[ia])) {
                if (EB) emit(false, ib);
                ++ib;
            } else {  // matched key-rank pair: A's copy
                if (EM) emit(true, ia);
                ++ia;
                ++ib;
            }
        }
    };
    KT rk[SET_STEPS];
    VT rv[VB > 0 ? SET_STEPS : 1];
    unsigned emitted = 0;
    int cnt = 0;
    if (regs) {  // one walk, outputs kept in registers (static slot per step)
        int ia = ia0, ib = ib0;
#pragma unroll
        for (int s = 0; s < SET_STEPS; ++s) {
            const bool ra = ia < ia1, rb = ib < ib1;
            if (ra || rb) {
                const KT ka = ra ? S.ka[ia] : KT(0), kb = rb ? S.kb[ib] : KT(0);
                bool e, fromA;
                if (ra && (!rb || ka < kb)) {
                    e = EA, fromA = true;
                } else if (rb && (!ra || kb < ka)) {
                    e = EB, fromA = false;
                } else {  // matched key-rank pair: A's copy
                    e = EM, fromA = true;
                    ++ib;
                }
                rk[s] = fromA ? ka : kb;
                if constexpr (VB > 0) rv[s] = fromA ? S.va[ia] : S.vb[ib];
                if (fromA) ++ia;
                else ++ib;
                if (e) {
                    emitted |= 1u << s;
                    ++cnt;
                }
            }
        }
    } else {
        walk([&](bool, int) { ++cnt; });
    }
    int tot;
    const int off = block_exclusive_sum<int, SET_NT / 32>(cnt, S.wsum, 1, &tot);
    // past the scan's barrier every thread has finished reading the windows:
    // the register path stages the tile's outputs over ka / va (warp 0 after
    // the look-back, so the tile's aggregate is published right after the scan)
    auto stage_out = [&]() {
        if (regs) {
            int p = off;
#pragma unroll
            for (int s = 0; s < SET_STEPS; ++s) {
                if ((emitted & (1u << s)) && p < SET_T + 2) {  // bound only binds on unsorted input
                    S.ka[p] = rk[s];
                    if constexpr (VB > 0) S.va[p] = rv[s];
                    ++p;
                }
            }
        }
    };
    if (tid >= 32) stage_out();
    if (tid < 32) {  // decoupled look-back over the tiles (warp 0, 32 predecessors per round)
        const int lane = tid;
        int64_t excl = 0;
        if (tile == 0) {
            if (lane == 0) {  // flag and value share one word: no fence needed
                atomicExch(reinterpret_cast<unsigned long long *>(&states[0]),
                           (unsigned long long)(ST_PRE | uint64_t(tot)));
            }
        } else {
            if (lane == 0)
                atomicExch(reinterpret_cast<unsigned long long *>(&states[tile]),
                           (unsigned long long)(ST_AGG | uint64_t(tot)));
            for (int pos = tile - 1;; pos -= 32) {
                const int k = pos - lane;
                uint64_t st = ST_PRE;  // virtual prefix 0 before tile 0
                if (k >= 0) {
                    do {
                        st = *reinterpret_cast<volatile uint64_t *>(&states[k]);
                    } while ((st & ~ST_VAL) == 0);  // predecessor not published yet
                }
                const unsigned pre = __ballot_sync(0xffffffffu, (st & ST_PRE) != 0);
                const int stop = pre ? __ffs(pre) - 1 : 32;  // nearest predecessor with a prefix
                int64_t v = lane <= stop ? int64_t(st & ST_VAL) : 0;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
                excl += v;
                if (pre) break;
            }
            if (lane == 0) {
                atomicExch(reinterpret_cast<unsigned long long *>(&states[tile]),
                           (unsigned long long)(ST_PRE | uint64_t(excl + tot)));
            }
        }
        if (lane == 0) {
            S.base = excl;
            if (tile == ntiles - 1) *nC = excl + tot;
        }
        stage_out();
    }
    __syncthreads();
    const int64_t base = S.base;
    if (regs) {  // coalesced store of the staged run
        const int nst = min(tot, SET_T + 2);
        for (int x = tid; x < nst && base + x < cap; x += SET_NT) {
            C[base + x] = S.ka[x];
            if constexpr (VB > 0) static_cast<VT *>(Cv)[base + x] = S.va[x];
        }
    } else {
        int64_t pos = base + off;
        walk([&](bool fromA, int x) {
            if (pos < cap) {
                C[pos] = fromA ? S.ka[x] : S.kb[x];
                if constexpr (VB > 0) static_cast<VT *>(Cv)[pos] = fromA ? S.va[x] : S.vb[x];
            }
            ++pos;
        });
    }
}

struct SetWs {
    Cut *cuts;
    uint64_t *states;
    unsigned *ticket;
    int64_t *nC;  // nC[0] result size, nC[1] contract-violation flag
    int64_t ntiles;
    size_t bytes;
};

SetWs carve(int64_t na, int64_t nb, void *ws, size_t bytes, bool *ok)
{
    SetWs w;
    const int64_t items = na + nb;
    w.ntiles = items > 0 ? ceil_div(items, SET_T) : 0;
    Carve cv(ws, bytes);
    w.ticket = cv.take<unsigned>(4);
    w.nC = cv.take<int64_t>(2);
    w.states = cv.take<uint64_t>(size_t(w.ntiles > 0 ? w.ntiles : 1));
    w.cuts = cv.take<Cut>(size_t(w.ntiles + 1));
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

template <typename KT, int VB, int OP>
msp_status launch_tiles(const void *A, const void *Av, int64_t na, const void *B, const void *Bv, int64_t nb,
                        const SetWs &w, void *C, void *Cv, int64_t cap, cudaStream_t s)
{
    auto kern = set_tile_kernel<KT, VB, OP>;
    const int smem = int(sizeof(SetSmem<KT, VB>));
    msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), smem, "set op: smem");
    if (st != MSP_OK) return st;
    kern<<<unsigned(w.ntiles), SET_NT, smem, s>>>(static_cast<const KT *>(A), Av, na, static_cast<const KT *>(B), Bv,
                                                  nb, w.cuts, w.ntiles, w.states, w.ticket, static_cast<KT *>(C), Cv,
                                                  cap, w.nC, reinterpret_cast<unsigned *>(w.nC + 1));
    return last_launch("set_tile_kernel");
}

template <typename KT, int VB>
msp_status launch_op(int op, const void *A, const void *Av, int64_t na, const void *B, const void *Bv, int64_t nb,
                     const SetWs &w, void *C, void *Cv, int64_t cap, cudaStream_t s)
{
    switch (op) {
    case 0: return launch_tiles<KT, VB, 0>(A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    case 1: return launch_tiles<KT, VB, 1>(A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    case 2: return launch_tiles<KT, VB, 2>(A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    default: return launch_tiles<KT, VB, 3>(A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    }
}

template <typename KT>
msp_status launch_kv(int op, int vb, const void *A, const void *Av, int64_t na, const void *B, const void *Bv,
                     int64_t nb, const SetWs &w, void *C, void *Cv, int64_t cap, cudaStream_t s)
{
    if (vb == 0) return launch_op<KT, 0>(op, A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    if (vb == 4) return launch_op<KT, 4>(op, A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    return launch_op<KT, 8>(op, A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
}

}  // namespace

size_t set_op_ws_bytes(int64_t na, int64_t nb)
{
    bool ok;
    return carve(na, nb, nullptr, SIZE_MAX, &ok).bytes + 256;
}

msp_status set_op_run(int op, const void *A, const void *Av, int64_t na, const void *B, const void *Bv, int64_t nb,
                      int key_bytes, int val_bytes, void *C, void *Cv, int64_t cap, int64_t *nC_host, int64_t *nC_dev,
                      void *ws, size_t ws_bytes, cudaStream_t s)
{
    bool ok;
    SetWs w = carve(na, nb, ws, ws_bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    if (nC_dev) w.nC = nC_dev;  // asynchronous form: the result words go to the caller's device buffer
    if (w.ntiles == 0) {
        if (nC_dev) return cuda_check(cudaMemsetAsync(nC_dev, 0, 2 * sizeof(int64_t), s), "set op: empty result");
        *nC_host = 0;
        return MSP_OK;
    }
    msp_status st;
    {
        const unsigned blocks = unsigned(std::min<int64_t>(ceil_div(w.ntiles + 1, 256), 148 * 8));
        if (key_bytes == 4)
            set_partition_kernel<uint32_t><<<blocks, 256, 0, s>>>(static_cast<const uint32_t *>(A), na,
                                                                  static_cast<const uint32_t *>(B), nb, w.ntiles, w.cuts,
                                                                  w.states, w.ticket, w.nC);
        else
            set_partition_kernel<uint64_t><<<blocks, 256, 0, s>>>(static_cast<const uint64_t *>(A), na,
                                                                  static_cast<const uint64_t *>(B), nb, w.ntiles, w.cuts,
                                                                  w.states, w.ticket, w.nC);
        st = last_launch("set_partition_kernel");
        if (st != MSP_OK) return st;
    }
    st = (key_bytes == 4) ? launch_kv<uint32_t>(op, val_bytes, A, Av, na, B, Bv, nb, w, C, Cv, cap, s)
                          : launch_kv<uint64_t>(op, val_bytes, A, Av, na, B, Bv, nb, w, C, Cv, cap, s);
    if (st != MSP_OK) return st;
    if (nC_dev) return MSP_OK;
    // the result size comes back through a pinned word (a pageable
    // destination would stage the 8-byte copy through a driver buffer)
    static thread_local int64_t *pinned = nullptr;
    if (!pinned) {
        st = cuda_check(cudaMallocHost(reinterpret_cast<void **>(&pinned), 2 * sizeof(int64_t)), "set op: pinned size");
        if (st != MSP_OK) {
            pinned = nullptr;
            return st;
        }
    }
    st = cuda_check(cudaMemcpyAsync(pinned, w.nC, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s), "set op: size");
    if (st != MSP_OK) return st;
    st = cuda_check(cudaStreamSynchronize(s), "set op: sync");
    if (st != MSP_OK) return st;
    *nC_host = pinned[0];
    if (pinned[1]) {
        set_error("set op: keys are not sorted ascending (as unsigned %d-byte integers)", key_bytes);
        return MSP_ERR_INPUT;
    }
    return MSP_OK;
}

}  // namespace msp
