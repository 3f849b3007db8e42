// query_reach.cu -- bit-lane batched reachability (sm_100a).
//
// Paper: reachability P(u, v) != {} (§2.1), the fourth benchmark problem
// (§5.1, Table 4), computed here on the transformed DAG of Alg. 1
// (departure nodes (v, tau), reading A11) with the GAC rounds of Alg. 3.
//
// One bit of state per (departure node, source): a sub-batch of up to 64 sources
// shares one u64 word per node, R[j] bit q = "query q can be at vertex v by time
// tau_j, having left x_q at >= alpha" -- instead of a 4-byte arrival per (vertex,
// query) in the EAT engine.  Every edge of a query batch is valid or not for all
// lanes at once (one window per call), so a relaxation is a word OR:
//   travel edge e = (j -> v, arrival a <= omega): VR[v] |= R[j]; R[snap(v, a)] |= R[j]
//   wait edges (v, tau_i) -> (v, tau_{i+1}): a prefix OR over v's node list
// Rounds: frontier = vertices with a node that gained bits ("dirty"; first/last
// dirty node per vertex).  k_reach_scan: a warp per dirty vertex runs the prefix OR
// over its nodes from the first dirty one (stopping past the last dirty node once
// the carry adds nothing), and expands the out-edges of every node whose word
// changed (occurrences of a node are contiguous: node_eoff); a relaxation whose
// tail node gains bits marks it dirty for the next round and, on a walked chain
// (>= walk_min edges), continues along the chain with the new bits (ChainEngine,
// P:L322-334).  Long edge ranges go to k_reach_big chunks.  Every OR is an atomicOr
// after a plain filter read: bits only grow, so a stale read is a subset.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include <cooperative_groups.h>

#include "tg_internal.cuh"

namespace cg = cooperative_groups;

namespace {

constexpr int RT = 256;
constexpr uint32_t RCHUNK = 256;  // edges per queued chunk
constexpr uint32_t RBIG = 128;    // a 32-node scan chunk with more changed out-edges queues them

struct ReachP {
    const uint32_t *vnode_off, *node_t, *node_eoff, *occ_slot, *occ_node, *slot_tn;
    const uint4 *occ_rch;
    const int4 *slots;
    const uint2 *lc;
    unsigned long long *R;   // [nnodes] node words
    unsigned long long *VR;  // [n] vertex words (output)
    uint32_t *D[2];          // dirty node bits by round parity
    uint32_t *dmin[2], *dmax[2];  // first / last dirty node per vertex by round parity
    uint32_t *vf[2];         // vertex frontier lists by round parity
    uint4 *bigq;             // {p0, p1, first node of the 32-node chunk, changed-node mask}
    uint64_t bigcap;
    RoundCtl *ctl;
    uint32_t round;
    uint32_t n, omega;
    unsigned long long *cnt;  // stats: [0] edge relaxations [1] node scans
    int stats;
};

// node j of vertex v gained bits in round P.round: it is scanned in round + 1
// Only the first-node atomicMin returns a value (it decides the vertex's single push);
// the dirty bit and the last dirty node are fire-and-forget reductions, so a relaxation
// waits on one atomic round trip, not on a chain of them.
__device__ __forceinline__ void mark_dirty(const ReachP &P, uint32_t j, uint32_t v) {
    const int o = (P.round + 1) & 1;
    atomicOr(P.D[o] + (j >> 5), 1u << (j & 31));
    atomicMax(P.dmax[o] + v, j);
    if (atomicMin(P.dmin[o] + v, j) == TG_NONE) {
        // one counter atomic per group of pushing lanes (a single-address counter hit by
        // every push serialises)
        cg::coalesced_group grp = cg::coalesced_threads();
        uint32_t k = 0;
        if (grp.thread_rank() == 0) k = atomicAdd(&P.ctl->cnt[(P.round + 1) & (TG_RING - 1)][0], grp.size());
        k = grp.shfl(k, 0) + grp.thread_rank();
        P.vf[o][k] = v;  // at most once per vertex per round: k < n
    }
}

// Relax out-occurrence p (sorted-edge position) of a node holding word w; walked
// chains continue with the bits their tail node gained.
__device__ __forceinline__ void reach_edge(const ReachP &P, uint32_t p, unsigned long long w) {
    // one coalesced 16-byte record {v, arrival | walked, tail node, tail tau}: a one-edge
    // (or not walked) chain needs nothing else
    const uint4 rc = __ldg(P.occ_rch + p);
    if ((rc.y & 0x7FFFFFFFu) > P.omega) return;  // arrival past the window: not valid
    if (!(rc.y >> 31)) {
        if (P.stats) atomicAdd(P.cnt + 0, 1ull);
        if (w & ~__ldcg(P.VR + rc.x)) atomicOr(P.VR + rc.x, w);
        if (rc.z == TG_NONE || rc.w >= P.omega) return;  // sink / nothing valid departs later
        // the filter read decides (bits only grow: a stale read can only add redundant
        // bits, which the OR absorbs and the next scan finds already present)
        const unsigned long long nb = w & ~__ldcg(P.R + rc.z);
        if (!nb) return;
        atomicOr(P.R + rc.z, nb);
        mark_dirty(P, rc.z, rc.x);
        return;
    }
    uint32_t s = __ldg(P.occ_slot + p);
    int4 sl = tg_ld_slot(P.slots + s);
    uint32_t s_end = s + 1;
    if ((uint32_t)sl.w != TG_SINGLE) {
        const uint2 info = __ldg(P.lc + (uint32_t)sl.w);
        s_end = info.x + info.y;
    }
    for (;;) {
        if (P.stats) atomicAdd(P.cnt + 0, 1ull);
        const uint32_t v = (uint32_t)sl.x;
        if (w & ~__ldcg(P.VR + v)) atomicOr(P.VR + v, w);
        const uint32_t tn = __ldg(P.slot_tn + s);
        if (tn == TG_NONE) return;  // sink: no later departure of v
        if (__ldg(P.node_t + tn) >= P.omega) return;  // nothing valid departs at >= omega
        const unsigned long long nb = w & ~__ldcg(P.R + tn);
        if (!nb) return;
        atomicOr(P.R + tn, nb);
        mark_dirty(P, tn, v);
        if (++s >= s_end) return;
        sl = tg_ld_slot(P.slots + s);  // the chain's next edge departs from node tn
        if ((uint32_t)sl.y > P.omega) return;
        w = nb;
    }
}

// Warp-cooperative scan of one dirty vertex with many departure nodes: prefix OR over
// the vertex's nodes (wait edges) 32 at a time from its first dirty node; out-edges of
// the nodes whose word changed are relaxed (or queued).
__device__ void scan_vertex_warp(const ReachP &P, int ib, uint32_t j0, uint32_t j1, uint32_t vend, uint32_t *big_cnt) {
    const int lane = threadIdx.x & 31;
    unsigned long long carry = 0;
    for (uint32_t jb = j0; jb < vend; jb += 32) {
        const uint32_t j = jb + lane;
        const bool valid = j < vend && __ldg(P.node_t + j) < P.omega;  // later nodes have no valid out-edge
        bool dirty = false;
        unsigned long long w = 0;
        if (valid) {
            const uint32_t bit = 1u << (j & 31);
            // this round's dirty bits were all set in the previous round (marks of this
            // round go to the other parity): a plain read decides, the clear is a RED
            if (j <= j1 && (__ldcg(P.D[ib] + (j >> 5)) & bit)) {
                dirty = true;
                atomicAnd(P.D[ib] + (j >> 5), ~bit);
            }
            w = __ldcg(P.R + j);
        }
        // inclusive prefix OR of the chunk's words, with the carry of earlier chunks
        unsigned long long incl = w;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl |= y;
        }
        unsigned long long excl = __shfl_up_sync(0xffffffffu, incl, 1);
        if (lane == 0) excl = 0;
        excl |= carry;
        const unsigned long long add = valid ? (excl & ~w) : 0ull;
        if (add) atomicOr(P.R + j, add);
        const bool changed = valid && (add != 0 || dirty);
        const unsigned long long nw_ = w | excl;  // the node's word after the wait edges
        carry = __shfl_sync(0xffffffffu, incl, 31) | carry;
        if (P.stats && lane == 0) atomicAdd(P.cnt + 1, (unsigned long long)min(32u, vend - jb));
        const uint32_t cm = __ballot_sync(0xffffffffu, changed);
        if (cm) {
            const uint32_t lo = __ffs(cm) - 1, hi = 31 - __clz(cm);
            const uint32_t p0 = __ldg(P.node_eoff + jb + lo), p1 = __ldg(P.node_eoff + jb + hi + 1);
            if (p1 - p0 > RBIG) {
                const uint32_t nch = (p1 - p0 + RCHUNK - 1) / RCHUNK;
                uint32_t k = 0;
                if (lane == 0) k = atomicAdd(big_cnt, nch);
                k = __shfl_sync(0xffffffffu, k, 0);
                for (uint32_t c = lane; c < nch; c += 32) {
                    const uint32_t b0 = p0 + c * RCHUNK, b1 = min(p1, b0 + RCHUNK);
                    if (k + c < P.bigcap) {
                        P.bigq[k + c] = make_uint4(b0, b1, jb, cm);
                    } else {
                        for (uint32_t p = b0; p < b1; p++) {
                            const uint32_t jn = __ldg(P.occ_node + p);
                            if ((cm >> (jn - jb)) & 1u) reach_edge(P, p, __ldcg(P.R + jn));
                        }
                    }
                }
            } else {
                for (uint32_t pb = p0; pb < p1; pb += 32) {
                    const uint32_t p = pb + lane;
                    const uint32_t jn = p < p1 ? __ldg(P.occ_node + p) : jb;
                    const uint32_t src = jn - jb;  // owner node's lane in this chunk
                    const unsigned long long ow = __shfl_sync(0xffffffffu, nw_, src);
                    if (p < p1 && ((cm >> src) & 1u)) reach_edge(P, p, ow);
                }
            }
        }
        if (!__shfl_sync(0xffffffffu, valid, 31)) break;  // past the window or the node list
        // past the last dirty node and the carry added nothing to the chunk's last
        // node: later nodes already hold it (prefix-closed, or dirty for next round)
        const bool last_ok = __shfl_sync(0xffffffffu, add == 0 && !dirty, 31);
        if (jb + 31 >= j1 && last_ok) break;
    }
}

// Round: warp per dirty vertex (a lane-per-vertex serial scan measured 1.7x slower:
// every node of a lane's vertex is a dependent step).
__global__ void __launch_bounds__(RT) k_reach_scan(ReachP P) {
    const int lane = threadIdx.x & 31;
    const uint32_t r = P.round;
    const int ib = r & 1;
    if (blockIdx.x == 0 && threadIdx.x < 4) P.ctl->cnt[(r + 2) & (TG_RING - 1)][threadIdx.x] = 0;  // two rounds ahead
    const uint32_t F = *(volatile uint32_t *)&P.ctl->cnt[r & (TG_RING - 1)][0];
    uint32_t *big_cnt = &P.ctl->cnt[r & (TG_RING - 1)][1];
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t i = gw; i < F; i += nw) {
        const uint32_t v = P.vf[ib][i];
        const uint32_t j0 = P.dmin[ib][v], j1 = P.dmax[ib][v];
        __syncwarp();
        if (lane == 0) { P.dmin[ib][v] = TG_NONE; P.dmax[ib][v] = 0; }
        scan_vertex_warp(P, ib, j0, j1, __ldg(P.vnode_off + v + 1), big_cnt);
    }
}

__global__ void __launch_bounds__(RT) k_reach_big(ReachP P) {
    const uint32_t r = P.round;
    const uint32_t B = (uint32_t)min((uint64_t)*(volatile uint32_t *)&P.ctl->cnt[r & (TG_RING - 1)][1], P.bigcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < B; it += nw) {
        const uint4 c = P.bigq[it];
        for (uint32_t p = c.x + lane; p < c.y; p += 32) {
            const uint32_t jn = __ldg(P.occ_node + p);
            if ((c.w >> (jn - c.z)) & 1u) reach_edge(P, p, __ldcg(P.R + jn));
        }
    }
}

// VInitial: VR[x_q] bit q; the first departure node of x_q at >= alpha gets bit q
// (the wait edges carry it to the later ones in round 1).
__global__ void k_reach_init(ReachP P, const uint32_t *srcs, uint32_t S, uint32_t alpha) {
    for (uint32_t q = threadIdx.x; q < S; q += blockDim.x) {
        const uint32_t x = srcs[q];
        const unsigned long long b = 1ull << q;
        atomicOr(P.VR + x, b);
        const uint32_t a = P.vnode_off[x], e = P.vnode_off[x + 1];
        const uint32_t j = tg_lower_bound(P.node_t, a, e, alpha);
        if (j < e && P.node_t[j] < P.omega) {
            atomicOr(P.R + j, b);
            mark_dirty(P, j, x);
        }
    }
}

// the bit-lane engine's occurrence records (built once per direction, on first use)
__global__ void k_reach_records(const uint2 *__restrict__ occ_rec, const uint32_t *__restrict__ occ_slot,
                                const uint32_t *__restrict__ slot_tn, const uint32_t *__restrict__ node_t, uint64_t m,
                                uint4 *__restrict__ out) {
    for (uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; p < m; p += (uint64_t)gridDim.x * blockDim.x) {
        const uint2 r = occ_rec[p];
        const uint32_t tn = slot_tn[occ_slot[p]];
        out[p] = make_uint4(r.x, r.y, tn, tn == TG_NONE ? 0xFFFFFFFFu : node_t[tn]);
    }
}

__global__ void k_reach_ctl(RoundCtl *ctl) {
    for (int i = 0; i < TG_RING; i++)
        for (int j = 0; j < 4; j++) ctl->cnt[i][j] = 0;
}

// out[q][v] = bit q of VR[v] (rows in the caller's vertex order)
__global__ void k_reach_extract(const unsigned long long *__restrict__ VR, uint32_t n, uint32_t S,
                                uint32_t *__restrict__ out, const uint32_t *__restrict__ perm) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const unsigned long long w = VR[perm ? perm[v] : v];
        for (uint32_t q = 0; q < S; q++) __stcs(out + (size_t)q * n + v, (uint32_t)((w >> q) & 1ull));
    }
}

}  // namespace

tg_status tg_run_reach_bits(tg_graph *g, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                            bool out_dev, cudaStream_t s) {
    ChainGraph &c = g->fwd;
    if (!c.occ_rch && g->m) {
        TG_TRY(c.arena.alloc((void **)&c.occ_rch, g->m * 16));
        TG_LAUNCH(k_reach_records, (unsigned)std::min<uint64_t>((g->m + 255) / 256, 148ull * 32), 256, 0, s, c.occ_rec,
                  c.occ_slot, c.slot_tn, c.node_t, g->m, c.occ_rch);
    }
    const uint64_t n = g->n, nn = c.nnodes;
    const uint32_t S = std::min<uint32_t>(64, k);
    ReachScratch &X = g->rs;
    if (!X.R || X.nn < nn || X.n < n) {
        TG_TRY_CUDA(cudaDeviceSynchronize());
        X.arena.free_all();
        X = ReachScratch{};
        X.nn = nn;
        X.n = n;
        DevArena &A = X.arena;
        const uint64_t dw = (nn + 31) / 32 + 1;
        TG_TRY(A.alloc((void **)&X.R, std::max<uint64_t>(nn, 1) * 8));
        TG_TRY(A.alloc((void **)&X.VR, n * 8));
        for (int i = 0; i < 2; i++) {
            TG_TRY(A.alloc((void **)&X.D[i], dw * 4));
            TG_TRY(A.alloc((void **)&X.dmin[i], n * 4));
            TG_TRY(A.alloc((void **)&X.dmax[i], n * 4));
            TG_TRY(A.alloc((void **)&X.vf[i], n * 4));
            TG_TRY_CUDA(cudaMemsetAsync(X.D[i], 0, dw * 4, s));
            TG_TRY_CUDA(cudaMemsetAsync(X.dmin[i], 0xFF, n * 4, s));
            TG_TRY_CUDA(cudaMemsetAsync(X.dmax[i], 0, n * 4, s));
        }
        X.bigcap = std::min<uint64_t>(g->m / RCHUNK + n / 8 + 4096, 1ull << 24);
        TG_TRY(A.alloc((void **)&X.bigq, X.bigcap * 16));
        TG_TRY(A.alloc((void **)&X.ctl, sizeof(RoundCtl)));
        TG_TRY(A.alloc((void **)&X.cnt, 64));
        TG_TRY(A.alloc((void **)&X.srcs, 64 * 4));
        TG_TRY(A.alloc((void **)&X.srcs_int, 64 * 4));
        TG_TRY(A.alloc((void **)&X.stage[0], 64 * n * 4));
        TG_TRY_CUDA(tg_pinned_get((void **)&X.h_ctr));
    }
    g->last = tg_query_stats{};
    const uint64_t launches0 = g_tg_launches;
    ReachP P{};
    P.vnode_off = c.vnode_off; P.node_t = c.node_t; P.node_eoff = c.node_eoff; P.occ_slot = c.occ_slot;
    P.occ_node = c.occ_node; P.slot_tn = c.slot_tn; P.slots = c.slots; P.lc = c.lc; P.occ_rch = c.occ_rch;
    P.R = X.R; P.VR = X.VR;
    for (int i = 0; i < 2; i++) { P.D[i] = X.D[i]; P.dmin[i] = X.dmin[i]; P.dmax[i] = X.dmax[i]; P.vf[i] = X.vf[i]; }
    P.bigq = X.bigq; P.bigcap = X.bigcap; P.ctl = X.ctl; P.n = g->n; P.omega = w.t_omega;
    P.cnt = X.cnt; P.stats = (int)g->opt_stats;
    const uint32_t grid = tg_grid_persistent(8);
    const int group = (int)std::max<int64_t>(1, g->opt_round_group);
    uint64_t relax_total = 0, scans_total = 0;
    for (uint32_t b0 = 0; b0 < k; b0 += S) {
        const uint32_t Sb = std::min(S, k - b0);
        TG_TRY(tg_load_sources_to(g, sources + b0, Sb, X.srcs, X.srcs_int, s));
        TG_TRY_CUDA(cudaMemsetAsync(X.R, 0, std::max<uint64_t>(nn, 1) * 8, s));
        TG_TRY_CUDA(cudaMemsetAsync(X.VR, 0, n * 8, s));
        if (P.stats) TG_TRY_CUDA(cudaMemsetAsync(X.cnt, 0, 64, s));
        TG_LAUNCH(k_reach_ctl, 1, 1, 0, s, X.ctl);
        uint32_t rounds = 0;
        P.round = 0;  // init pushes into round 1's frontier
        TG_LAUNCH(k_reach_init, 1, 64, 0, s, P, X.srcs_int, Sb, w.t_alpha);  // sources reach themselves
        if (g->m > 0 && w.t_alpha < w.t_omega) {
            uint32_t r = 1;
            for (;;) {
                for (int i = 0; i < group; i++, r++) {
                    P.round = r;
                    TG_LAUNCH_RELAX(k_reach_scan, grid, RT, 0, s, P);
                    TG_LAUNCH_RELAX(k_reach_big, grid, RT, 0, s, P);
                }
                TG_TRY_CUDA(cudaMemcpyAsync(X.h_ctr, X.ctl, sizeof(RoundCtl), cudaMemcpyDeviceToHost, s));
                TG_TRY_CUDA(cudaStreamSynchronize(s));
                const RoundCtl *h = (const RoundCtl *)X.h_ctr;
                // r is the next round: its frontier count was written by the rounds just run
                if (h->cnt[r & (TG_RING - 1)][0] == 0) {
                    // the group's first round with an empty frontier did no work
                    rounds = r - 1;
                    for (uint32_t q = r + 1 - (uint32_t)group; q < r; q++)
                        if (h->cnt[q & (TG_RING - 1)][0] == 0) { rounds = q - 1; break; }
                    break;
                }
                if (r > 10000000) { tg_set_error("reach rounds did not converge"); return TG_ERR_CUDA; }
            }
        }
        g->last.rounds = std::max(g->last.rounds, rounds);
        g->last.sub_batches++;
        uint32_t *o = out_dev ? out + (size_t)b0 * n : X.stage[0];
        TG_LAUNCH(k_reach_extract, (unsigned)std::min<uint64_t>((n + 255) / 256, 148ull * 8), 256, 0, s, X.VR,
                  g->n, Sb, o, g->relabeled ? g->perm : (const uint32_t *)nullptr);
        if (!out_dev)
            TG_TRY_CUDA(cudaMemcpyAsync(out + (size_t)b0 * n, X.stage[0], (size_t)Sb * n * 4, cudaMemcpyDeviceToHost, s));
        if (P.stats) {
            unsigned long long h[2];
            TG_TRY_CUDA(cudaMemcpyAsync(h, X.cnt, 16, cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
            relax_total += h[0];
            scans_total += h[1];
        }
    }
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    g->last.slots_relaxed = relax_total;
    g->last.slots_union = scans_total;  // bit-lane engine: node scans (reported in the same field)
    g->last.kernel_launches = g_tg_launches - launches0;
    return TG_OK;
}
