// sweep_ws.cuh -- warp-specialised directional sweep (same tiles, ring layout and per-interface
// arithmetic as k_sweep_s in sweep.cuh, so results are bitwise the same).
//
// k_sweep_s keeps its staging inside each warp: per step it waits for its own cp.async
// copies, computes the primitives of the newest chunk (rcp / sqrt / rsqrt chains) and only then
// starts the interface setup -- latency that two warps per scheduler cannot cover (
// proxy with staging and primitives removed: -8 % per 512^3 stage).  Here a CTA holds 8 consumer
// warps (2 warpgroups) that only evaluate interface fluxes and 4 producer warps (1 warpgroup) that
// fill the consumers' rings: producer p serves consumers p and p + 4, copying their chunks with
// cp.async one chunk ahead and computing the primitives of each landed chunk.  Register budgets
// are rebalanced with setmaxnreg (consumers WS_CREG, producers WS_PREG; 8 * WS_CREG + 4 *
// WS_PREG = 12 * 168).  Each consumer ring has NSLOT = NR / WS chunk slots, each with a `full`
// (32 producer-lane arrivals: copies landed + primitives stored) and an `empty` mbarrier (32
// consumer-lane arrivals after the step that last reads the chunk).
#pragma once
#include "sweep.cuh"

namespace crocco {

constexpr int WS_CONS = 8;                          // consumer warps per CTA
constexpr int WS_PROD = 4;                          // producer warps per CTA
constexpr int WS_THREADS = 32 * (WS_CONS + WS_PROD);
#ifndef WS_CREG
#define WS_CREG 224
#endif
#ifndef WS_PREG
#define WS_PREG 56
#endif
static_assert(WS_CONS * WS_CREG + WS_PROD * WS_PREG <= (WS_CONS + WS_PROD) * 168, "register budget");

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, unsigned cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
    asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.release.cta.shared::cta.b64 st, [%0];\n}\n" ::"r"(smem_u32(b))
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, unsigned parity) {
    asm volatile(
        "{\n .reg .pred p;\n WAIT_%=:\n"
        " mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(b)),
        "r"(parity)
        : "memory");
}

// geometry of one work unit (a line segment of a warp tile) for one lane
struct WsGeo {
    int e0, e1, qbase, qmax, nsteps;
    int ci, cj, ck;
    bool lvalid, xcv;
    int64_t cpo, cpv, xco;
};
template <int D, bool VISC>
__device__ __forceinline__ bool ws_geo(const SweepArgs &a, const Lay &L, int64_t gw, int lane, WsGeo &g) {
    using RG = RingGeom<D, VISC>;
    constexpr int C = RG::C, WS = RG::WS;
    const int lt = (D == 0) ? (lane >> 3) : (lane & 7);
    const int nd = D == 0 ? L.n0 : (D == 1 ? L.n1 : L.n2);
    const int nseg = (nd + a.seg - 1) / a.seg;
    int64_t ntl;
    if (D == 0) ntl = ((int64_t)L.n1 * L.n2 + C - 1) / C;
    else ntl = (int64_t)((L.n0 + C - 1) / C) * ((D == 1) ? L.n2 : L.n1);
    if (gw >= ntl * nseg) return false;
    const int sg = (int)(gw / ntl);
    const int64_t r = gw % ntl;
    g.e0 = sg * a.seg;
    g.e1 = min(nd, g.e0 + a.seg);
    g.qbase = g.e0 - 3 - RG::QOFF;
    g.nsteps = (g.e1 - g.e0 + 1 + WS - 1) / WS;
    g.qmax = nd + G - 1 - g.qbase;
    g.ci = g.cj = g.ck = 0;
    g.cpo = g.cpv = g.xco = 0;
    g.xcv = false;
    if (D == 0) {
        const int64_t t = r * C + lt, nl = (int64_t)L.n1 * L.n2;
        g.lvalid = t < nl;
        if (g.lvalid) {
            g.cj = (int)(t % L.n1);
            g.ck = (int)(t / L.n1);
        }
        const int64_t tc = r * C + (lane & 3);
        g.xcv = tc < nl;
        if (g.xcv) g.xco = at(L, 0, (int)(tc % L.n1), (int)(tc / L.n1));
    } else {
        const int tiles = (L.n0 + C - 1) / C;
        const int colbase = (int)(r % tiles) * C, oo = (int)(r / tiles);
        g.ci = colbase + lt;
        g.lvalid = g.ci < L.n0;
        if (D == 1) g.ck = oo;
        else g.cj = oo;
        const int gi = colbase + 2 * (lane & 3);
        g.cpo = D == 1 ? at(L, gi, 0, oo) : at(L, gi, oo, 0);
        g.cpv = D == 1 ? vat(a.V, gi, 0, oo) : vat(a.V, gi, oo, 0);
    }
    return true;
}

// copies of chunk `ch` of a consumer's ring (lane mapping of k_sweep_s's issue)
template <int D, bool VISC>
__device__ __forceinline__ void ws_issue(const SweepArgs &a, const Lay &L, const WsGeo &g, double *sv, int lane,
                                         int ch) {
    using RG = RingGeom<D, VISC>;
    constexpr int WS = RG::WS, C = RG::C, NR = RG::NR, VS = RG::VS;
    const double *Mrow = a.in.M + (int64_t)(1 + 3 * D) * L.cs;
    if (D == 0) {
        const int col = lane & 3, pr = (lane >> 2) & 3, vg = lane >> 4;
        const int q = ch * WS + 2 * pr, gq = g.qbase + q;
        if (g.xcv && q <= g.qmax) {
            double *dst = sv + RG::slot(q, col);
#pragma unroll
            for (int t = 0; t < 4; t++) {
                const int v = 4 * vg + t;
                const double *src = (v < 5 ? a.in.U + v * L.cs : Mrow + (v - 5) * L.cs) + g.xco + gq;
                if ((g.e0 & 1) == 0) {
                    cp_async16(dst + v * VS, src);
                } else {
                    cp_async8(dst + v * VS, src);
                    if (q + 1 <= g.qmax) cp_async8(dst + v * VS + 1, src + 1);
                }
            }
        }
    } else {
        constexpr int SV_FV_ = SV_FV;
        const int64_t sst = D == 1 ? L.py : L.pz;
        const int64_t vst = D == 1 ? a.V.py : a.V.pz;
        const int nd = D == 1 ? L.n1 : L.n2;
        const int v = lane >> 2;
        const double *src0 = v < 5 ? a.in.U + v * L.cs + g.cpo : Mrow + (v - 5) * L.cs + g.cpo;
        double *dst0 = sv + v * VS + 2 * (lane & 3);
#pragma unroll
        for (int pt = 0; pt < WS; pt++) {
            const int q = ch * WS + pt, gq = g.qbase + q;
            if (q <= g.qmax) cp_async16(dst0 + (q & (NR - 1)) * C, src0 + gq * sst);
        }
        if (VISC && v < 4) {
            const double *srcf = a.in.FV + v * a.in.vcs + g.cpv;
            double *dstf = sv + (SV_FV_ + v) * VS + 2 * (lane & 3);
#pragma unroll
            for (int pt = 0; pt < WS; pt++) {
                const int q = ch * WS + pt, gq = g.qbase + q;
                if (q <= g.qmax && gq >= -2 && gq <= nd + 1) cp_async16(dstf + (q & (NR - 1)) * C, srcf + gq * vst);
            }
        }
    }
}

// primitives of chunk `ch` (one point per lane), from the staged state (k_sweep_s's prims)
template <int D, bool VISC>
__device__ __forceinline__ void ws_prims(const Phys &ph, const WsGeo &g, double *sv, int lane, int ch) {
    using RG = RingGeom<D, VISC>;
    constexpr int WS = RG::WS, VS = RG::VS, SV_P = sv_p(VISC);
    const int ls = (D == 0) ? (lane & 7) : (lane >> 3);
    const int lt = (D == 0) ? (lane >> 3) : (lane & 7);
    const int q = ch * WS + ls;
    if (q > g.qmax) return;
    double *bq = sv + RG::slot(q, lt);
    const double rho = bq[0], ru = bq[VS], rv = bq[2 * VS], rw = bq[3 * VS], E = bq[4 * VS];
    const double ir = rcp_nr(rho);
    const double u = ru * ir, v = rv * ir, w = rw * ir;
    const double pr = ph.gm1 * fma(-0.5, fma(ru, u, fma(rv, v, rw * w)), E);
    bq[(SV_P + PU) * VS] = u;
    bq[(SV_P + PV) * VS] = v;
    bq[(SV_P + PW) * VS] = w;
    bq[(SV_P + PP) * VS] = pr;
    bq[(SV_P + PC) * VS] = sqrt_nr(ph.gamma * pr * ir);
    bq[(SV_P + PIS) * VS] = rsqrt_nr(rho);
    bq[(SV_P + PH) * VS] = (E + pr) * ir;
}

template <int D, bool VISC>
struct WsGeomSm {
    static constexpr int NSLOT = RingGeom<D, VISC>::NR / RingGeom<D, VISC>::WS;  // chunk slots per ring
    static constexpr size_t BAR_OFF = (size_t)WS_CONS * RingGeom<D, VISC>::PER_WARP;  // doubles
    static constexpr size_t BYTES = (BAR_OFF + (size_t)WS_CONS * NSLOT * 2) * sizeof(double);
};

template <int D, bool VISC, bool LIM>
__global__ void __launch_bounds__(WS_THREADS, 1) k_sweep_ws(const __grid_constant__ SweepArgs a, const Lay L,
                                                           const Phys ph) {
    using RG = RingGeom<D, VISC>;
    using SG = WsGeomSm<D, VISC>;
    constexpr int WS = RG::WS, NR = RG::NR, LA = RG::LA, VS = RG::VS, C = RG::C;
    constexpr int NSLOT = SG::NSLOT;
    static_assert(NSLOT >= LA + 2, "ring slots");
    static_assert(D != 0 || !VISC, "the xi sweep carries no viscous interface term");
    extern __shared__ double smem_dyn[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem_dyn + SG::BAR_OFF);  // [consumer][full 0..NSLOT-1, empty ..]
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x < WS_CONS * NSLOT * 2) mbar_init(bars + threadIdx.x, 32);
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    __syncthreads();

    if (warp >= WS_CONS) {
        // ---------------- producer warpgroup ----------------
        asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;\n" ::"n"(WS_PREG));
        const int p = warp - WS_CONS;
        WsGeo g0, g1;
        const int64_t gw0 = (int64_t)blockIdx.x * WS_CONS + p, gw1 = gw0 + WS_PROD;
        const int n0 = ws_geo<D, VISC>(a, L, gw0, lane, g0) ? g0.nsteps + LA : 0;
        const int n1 = ws_geo<D, VISC>(a, L, gw1, lane, g1) ? g1.nsteps + LA : 0;
        double *sv0 = smem_dyn + (size_t)p * RG::PER_WARP, *sv1 = smem_dyn + (size_t)(p + WS_PROD) * RG::PER_WARP;
        uint64_t *b0 = bars + p * 2 * NSLOT, *b1 = bars + (p + WS_PROD) * 2 * NSLOT;
        const int nm = max(n0, n1);
        // second version: K chunks in flight; the primitives of chunk ch are published BEFORE
        // waiting for the slot of chunk ch + K (released by consumer step ch + K - NSLOT <= ch - LA - 1)
        constexpr int K = NSLOT - LA - 1;
        static_assert(K >= 1 && K <= 2, "lookahead");
#pragma unroll
        for (int c = 0; c < K; c++) {
            if (c < n0) ws_issue<D, VISC>(a, L, g0, sv0, lane, c);
            if (c < n1) ws_issue<D, VISC>(a, L, g1, sv1, lane, c);
            cp_async_commit();
        }
        for (int ch = 0; ch < nm; ch++) {
            if constexpr (K == 1) asm volatile("cp.async.wait_group 0;\n" ::: "memory");  // chunk ch landed
            else asm volatile("cp.async.wait_group 1;\n" ::: "memory");
            __syncwarp();
            if (ch < n0) {
                ws_prims<D, VISC>(ph, g0, sv0, lane, ch);
                mbar_arrive(b0 + ch % NSLOT);
            }
            if (ch < n1) {
                ws_prims<D, VISC>(ph, g1, sv1, lane, ch);
                mbar_arrive(b1 + ch % NSLOT);
            }
            const int nx = ch + K, s = nx % NSLOT;
            const unsigned par = ((unsigned)(nx / NSLOT) + 1u) & 1u;  // completion nx/NSLOT - 1 of empty[s]
            if (nx < n0) {
                if (nx >= NSLOT) mbar_wait(b0 + NSLOT + s, par);
                ws_issue<D, VISC>(a, L, g0, sv0, lane, nx);
            }
            if (nx < n1) {
                if (nx >= NSLOT) mbar_wait(b1 + NSLOT + s, par);
                ws_issue<D, VISC>(a, L, g1, sv1, lane, nx);
            }
            cp_async_commit();
        }
        cp_async_wait_all();
        return;
    }

    // ---------------- consumer warps ----------------
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;\n" ::"n"(WS_CREG));
    constexpr int SV_P = sv_p(VISC);
    (void)SV_P;
    WsGeo g;
    const int64_t gw = (int64_t)blockIdx.x * WS_CONS + warp;
    if (!ws_geo<D, VISC>(a, L, gw, lane, g)) return;
    double *sv = smem_dyn + (size_t)warp * RG::PER_WARP;
    uint64_t *bf = bars + warp * 2 * NSLOT, *be = bf + NSLOT;
    double *cb = sv + RG::SVN * VS + lane;  // this lane's prefetched operands
    const int ls = (D == 0) ? (lane & 7) : (lane >> 3);
    const int lt = (D == 0) ? (lane >> 3) : (lane & 7);
    (void)C;
    const bool inv = a.inv != 0;
    const int e0 = g.e0, e1 = g.e1;
    const int64_t sst = D == 0 ? 1 : (D == 1 ? L.py : L.pz);
    const int64_t rstep = (D == 0 ? 1 : (D == 1 ? (int64_t)L.n0 : (int64_t)L.n0 * L.n1)) * WS;
    const int64_t pstep = sst * WS;
    int64_t rr, pp;
    {
        const int e = e0 - 1 + ls;
        const int pi = D == 0 ? e : g.ci, pj = D == 1 ? e : g.cj, pk = D == 2 ? e : g.ck;
        rr = (int64_t)pi + (int64_t)L.n0 * (pj + (int64_t)L.n1 * pk);
        pp = at(L, pi, pj, pk);
    }
#pragma unroll
    for (int ch = 0; ch < LA; ch++) mbar_wait(bf + ch, 0u);
    double F[5], Fc[5];
#pragma unroll
    for (int c = 0; c < 5; c++) Fc[c] = 0.0;
    for (int st = 0; st < g.nsteps; st++, rr += rstep, pp += pstep) {
        {
            const int ch = st + LA;
            mbar_wait(bf + ch % NSLOT, (unsigned)(ch / NSLOT) & 1u);
        }
        const int e = e0 - 1 + WS * st + ls;  // this lane's interface e+1/2
        const bool act = g.lvalid && e <= e1 - 1;
        const bool own = act && e >= e0;      // this lane finishes point e
        const SAcc<NR, C, VISC, RG::CS> A{sv, WS * st + ls + RG::QOFF, lt};
        if (own && a.mode != 0) {             // accumulate / update operands
#pragma unroll
            for (int c = 0; c < 5; c++)
                if (c > 0 || a.mode != 4) cp_async8(cb + 32 * c, a.R + c * a.rcs + rr);
            if (a.mode == 2 || a.mode == 3) {
                cp_async8(cb + 32 * 5, a.in.M + pp);
                if (a.mode == 3) {
#pragma unroll
                    for (int c = 0; c < 5; c++) {
                        if (a.stage != 0) cp_async8(cb + 32 * (6 + c), a.dU + c * L.cs + pp);
                    }
                }
            }
        }
        cp_async_commit();
        if (act) {
            FluxSetup su;
            if (inv) flux_setup(A, ph, su);
            flux_fields<D, SAcc<NR, C, VISC, RG::CS>, LIM>(A, su, inv, VISC, ph, F);
        } else {
#pragma unroll
            for (int c = 0; c < 5; c++) F[c] = 0.0;
        }
        double dF[5];
        if constexpr (RG::CARRY) {
            double *fs = sv + RG::SVN * VS + RG::NCB * 32;
            double *cur = fs + (st & 1) * 160, *prv = fs + ((st & 1) ^ 1) * 160;
#pragma unroll
            for (int c = 0; c < 5; c++) cur[32 * c + lane] = F[c];
            __syncwarp();
            const int src = ls != 0 ? (D == 0 ? lane - 1 : lane - 8) : (D == 0 ? (lane | 7) : 24 + lt);
            const double *from = ls != 0 ? cur : prv;
#pragma unroll
            for (int c = 0; c < 5; c++) {
                const double Fm = st == 0 && ls == 0 ? 0.0 : from[32 * c + src];
                dF[c] = Fm - F[c];
            }
        } else {
#pragma unroll
            for (int c = 0; c < 5; c++) {
                double Fm;
                if (D == 0) {
                    Fm = __shfl_up_sync(0xffffffffu, F[c], 1, 8);
                    if (ls == 0) Fm = Fc[c];
                    Fc[c] = __shfl_sync(0xffffffffu, F[c], 7, 8);
                } else {
                    Fm = __shfl_up_sync(0xffffffffu, F[c], 8);
                    if (ls == 0) Fm = Fc[c];
                    Fc[c] = __shfl_sync(0xffffffffu, F[c], 24 + lt);
                }
                dF[c] = Fm - F[c];
            }
        }
        cp_async_wait_all();  // own operands landed
        if (own) {
            if (a.mode == 0) {
#pragma unroll
                for (int c = 0; c < 5; c++) a.R[c * a.rcs + rr] = dF[c];
            } else {
                double Rt[5];
#pragma unroll
                for (int c = 0; c < 5; c++) Rt[c] = (c == 0 && a.mode == 4) ? dF[0] : cb[32 * c] + dF[c];
                if (a.mode == 1 || a.mode == 4) {
#pragma unroll
                    for (int c = 0; c < 5; c++) a.R[c * a.rcs + rr] = Rt[c];
                } else if (a.mode == 2) {
                    const double J = cb[32 * 5];
#pragma unroll
                    for (int c = 0; c < 5; c++) a.rhs[c * L.cs + pp] = J * Rt[c];
                } else {
                    const double J = cb[32 * 5];
#pragma unroll
                    for (int c = 0; c < 5; c++) {
                        const double rv = J * Rt[c];
                        const double du = (a.stage == 0) ? a.dt * rv : fma(a.A, cb[32 * (6 + c)], a.dt * rv);
                        a.dU[c * L.cs + pp] = du;
                        a.Uout[c * L.cs + pp] = fma(a.B, du, A.U(2, c));
                    }
                }
            }
        }
        mbar_arrive(be + st % NSLOT);  // chunk st is not read by later steps
    }
}

}  // namespace crocco
