// sweep.cuh -- directional sweeps (WENOx, WENOy, WENOz + Viscous)
// fused with the RHS assembly and the RK Update.
//
// Work decomposition (one warp = 32 interfaces per step, each interface flux
// evaluated exactly once; the point difference uses the neighbour interface
// exchanged by warp shuffle, the step-to-step carry stays in registers):
//   D = 0 (xi, contiguous): a warp holds 4 lines x 8 consecutive interfaces and
//     advances 8 interfaces per step.
//   D = 1, 2 (eta, zeta): a warp holds 8 consecutive i (64-B coalesced rows) x 4
//     consecutive interfaces and advances 4 per step.
//   A line is marched over segments of `seg` points; each segment recomputes
//   the one interface it shares with the previous segment.
// Every interface, in any decomposition and any lane, runs the same code
// (flux_setup + flux_fields), so an n-block run equals the 1-block run bit for bit.
//
// Accumulation of R = -sum_d (F_{i+1/2} - F_{i-1/2}) per point in fixed order
// xi, eta, zeta (mode 0 writes, mode 1 adds); the zeta sweep finishes the point:
//   mode 2: rhs = J R ;  mode 3: dU <- A dU + dt J R, U_out = U_in + B dU.
#pragma once
#include "common.cuh"
#include "flux.cuh"

namespace crocco {

// bit D: sweep D passes neighbour / carried interface fluxes through shared memory instead of a
// register carry (round 1: eta -4 %, xi +16 %, zeta 0; re-measured at the end of round 2 on the final
// kernels together with the lambda trees of flux.cuh: all three directions, -0.45 ms per 512^3 stage,
// profiles/r02_variants_retune_final.jsonl)
constexpr int CARRY_SMEM = 7;
// threads per CTA and min CTAs per SM of sweep D: 4 warps, register-limited to 2 CTAs (8 warps)
// per SM at 253 registers.  Measured (profiles/r02_variants_sweep.jsonl): capping the
// registers for 10 or 12 warps per SM (2-warp CTAs) spills 150-280 B/thread and runs 25 % slower.
__host__ __device__ constexpr int sweep_threads(int) { return 128; }
__host__ __device__ constexpr int sweep_minb(int) { return 1; }

struct SweepArgs {
    FluxIn in;
    VLay V;
    double *R;          // accumulator, compact interior layout i + n0 (j + n1 k)
    int64_t rcs;        // its component stride
    int inv, visc;      // terms evaluated in this direction
    int mode;           // 0 write R, 1 add to R, 2 rhs = J R, 3 RK update,
                        // 4 add to the viscous divergence in R comps 1..4 (k_visc_tiled), write comp 0
    int seg;            // march segment
    double *rhs;        // mode 2 (padded layout)
    const double *Uin;  // mode 3 (padded layout): must be the swept state in.U (its values are read from the ring)
    double *Uout, *dU;
    double A, B, dt;
    int stage;
};

// ---------------------------------------------------------------------------
// Shared-memory staged sweep: each warp
// keeps a ring of its stencil window in shared memory -- conserved state and
// metric row copied with cp.async one step ahead of use, primitives computed
// once per point when it enters the ring -- so the characteristic WENO reads
// only shared memory.  Warps are independent (no block barriers).
// ---------------------------------------------------------------------------

template <int D, bool VISC>
struct RingGeom {
    static constexpr int WS = (D == 0) ? 8 : 4;    // interfaces per step
    static constexpr int C = 32 / WS;              // columns (lines) per warp
    static constexpr int LA = (D == 0) ? 1 : 2;    // chunks ahead needed by a step
    static constexpr int NR = (D == 0) ? 32 : 16;  // ring points (>= (LA + 2) * WS, power of 2)
    static_assert(NR >= (LA + 2) * WS && (NR & (NR - 1)) == 0, "ring too small");
    static constexpr int SVN = sv_n(VISC);         // staged values per ring point
    // xi: column-major ring (16-B copies of point pairs along the line); column stride padded 32 -> 40
    static constexpr int CS = D == 0 ? NR + 8 : 0;
    static constexpr int VS = CS ? C * CS : NR * C;  // doubles per staged value
    static constexpr int QOFF = D == 0 ? 1 : 0;      // xi: ring point 0 is swept index e0 - 4 (even)
    __host__ __device__ static constexpr int slot(int q, int col) {
        return CS ? col * CS + (q & (NR - 1)) : (q & (NR - 1)) * C + col;
    }
    // prefetched accumulate / update operands per lane: xi (mode 0 / 4) and eta (mode 1) read R;
    // zeta finishes the point (mode 2: R, J; mode 3: R, J, dU -- U_in comes from the ring)
    static constexpr int NCB = D == 2 ? 11 : 5;
    static constexpr bool CARRY = (CARRY_SMEM >> D) & 1;
    static constexpr int NFC = CARRY ? 2 * 5 * 32 : 0;  // interface fluxes of two steps
    static constexpr int PER_WARP = SVN * VS + NCB * 32 + NFC;  // doubles
};

// MODE = SweepArgs::mode as a template parameter: each launch compiles only its own accumulate / update
// path (a run-time mode let every direction's kernel carry all five, and their register allocation)
// INV: 1 inviscid flux on, 0 off (dir_mask / terms), 2 decided at run time by a.inv (the limiter
// variants: a compile-time 1 makes ptxas spill their eta sweep, measured 19.1 vs 13.3 ms per 512^3 launch)
template <int D, bool VISC, bool LIM, int MODE, int INV = 1>
__global__ void __launch_bounds__(sweep_threads(D), sweep_minb(D)) k_sweep_s(const __grid_constant__ SweepArgs a,
                                                                          const Lay L, const Phys ph) {
    using RG = RingGeom<D, VISC>;
    constexpr int WS = RG::WS, C = RG::C, LA = RG::LA, NR = RG::NR;
    constexpr int VS = RG::VS;
    constexpr int SV_P = sv_p(VISC);
    static_assert(D != 0 || !VISC, "the xi sweep carries no viscous interface term");
    extern __shared__ double smem_dyn[];
    const int lane = threadIdx.x & 31;
    double *sv = smem_dyn + (threadIdx.x >> 5) * RG::PER_WARP;
    double *cb = sv + RG::SVN * VS + lane;  // this lane's prefetched operands
    const int ls = (D == 0) ? (lane & 7) : (lane >> 3);  // sweep offset of this lane
    const int lt = (D == 0) ? (lane >> 3) : (lane & 7);  // column of this lane
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const bool inv = INV == 2 ? a.inv != 0 : INV == 1;
    const int nd = D == 0 ? L.n0 : (D == 1 ? L.n1 : L.n2);
    const int nseg = (nd + a.seg - 1) / a.seg;
    int64_t ntl;
    if (D == 0) ntl = ((int64_t)L.n1 * L.n2 + C - 1) / C;
    else ntl = (int64_t)((L.n0 + C - 1) / C) * ((D == 1) ? L.n2 : L.n1);
    if (gw >= ntl * nseg) return;
    const int sg = (int)(gw / ntl);
    const int64_t r = gw % ntl;
    const int e0 = sg * a.seg, e1 = min(nd, e0 + a.seg);
    const int qbase = e0 - 3 - RG::QOFF;             // swept index of ring point q = 0
    const int nsteps = (e1 - e0 + 1 + WS - 1) / WS;  // interfaces e0-1 .. e1-1
    const int qmax = nd + G - 1 - qbase;             // last ring point inside the padded box
    const int64_t sst = D == 0 ? 1 : (D == 1 ? L.py : L.pz);  // swept strides
    const int64_t vst = D == 0 ? 1 : (D == 1 ? a.V.py : a.V.pz);

    // this lane's own line (for its interfaces) ...
    int ci = 0, cj = 0, ck = 0;
    bool lvalid;
    // ... and the line / column it copies for the ring (D = 0: column lane>>3; D != 0: pair lane&3)
    int64_t cpo = 0, cpv = 0;  // padded / FV-box index of the copy column at swept index 0
    bool cvalid;
    if (D == 0) {
        const int64_t t = r * C + lt, nl = (int64_t)L.n1 * L.n2;
        lvalid = cvalid = t < nl;
        if (lvalid) {
            cj = (int)(t % L.n1);
            ck = (int)(t / L.n1);
        }
        cpo = at(L, 0, cj, ck);
        cpv = vat(a.V, 0, cj, ck);
    } else {
        const int tiles = (L.n0 + C - 1) / C;
        const int colbase = (int)(r % tiles) * C, oo = (int)(r / tiles);
        ci = colbase + lt;
        lvalid = ci < L.n0;
        if (D == 1) ck = oo;
        else cj = oo;
        cvalid = true;  // whole 8-column rows are copied (columns past n0 stay in the row padding)
        const int gi = colbase + 2 * (lane & 3);
        cpo = D == 1 ? at(L, gi, 0, oo) : at(L, gi, oo, 0);
        cpv = D == 1 ? vat(a.V, gi, 0, oo) : vat(a.V, gi, oo, 0);
    }
    const double *Mrow = a.in.M + (int64_t)(1 + 3 * D) * L.cs;
    // xi copies: line (column) lane & 3 of this warp
    bool xcv = false;
    int64_t xco = 0;
    if (D == 0) {
        const int64_t t = r * C + (lane & 3);
        xcv = t < (int64_t)L.n1 * L.n2;
        if (xcv) xco = at(L, 0, (int)(t % L.n1), (int)(t / L.n1));
    }

    // issue the copies of chunk `ch`: U (5) + metric row (3) [+ FV (4)] of WS points x C columns
    // (predicated cp.async: points outside the padded box / FV box are zero-filled, nothing read, no
    // branch; measured with the xi / eta group-A predication -0.7 ms per 512^3 stage)
    auto issue = [&](int ch) {
        if (D == 0) {
            // xi, column-major ring: 16-B copies of point pairs (2p, 2p+1) -- lane: column lane&3,
            // pair (lane>>2)&3, values 4 (lane>>4) .. 4 (lane>>4) + 3 (U 0-4, metric row 5-7);
            // 8-B copies when the segment start is odd (16-B source alignment)
            const int col = lane & 3, pr = (lane >> 2) & 3, vg = lane >> 4;
            const int q = ch * WS + 2 * pr, gq = qbase + q;
            {
                const bool ok = xcv && q <= qmax, ok1 = ok && q + 1 <= qmax;
                double *dst = sv + RG::slot(q, col);
#pragma unroll
                for (int t = 0; t < 4; t++) {
                    const int v = 4 * vg + t;
                    const double *base = v < 5 ? a.in.U + v * L.cs : Mrow + (v - 5) * L.cs;
                    const double *src = ok ? base + xco + gq : base;
                    if ((e0 & 1) == 0) {
                        cp_async16z(dst + v * VS, src, ok);
                    } else {
                        cp_async8z(dst + v * VS, src, ok);
                        cp_async8z(dst + v * VS + 1, ok1 ? src + 1 : base, ok1);
                    }
                }
            }
        } else {
            // lane: value lane>>2 (U0-4, M0-2) [and FV lane>>2 for lanes < 16] of the
            // column pair lane&3, all WS points, 16-B copies
            const int v = lane >> 2;
            const double *src0 = v < 5 ? a.in.U + v * L.cs + cpo : Mrow + (v - 5) * L.cs + cpo;
            double *dst0 = sv + v * VS + 2 * (lane & 3);
#pragma unroll
            for (int pt = 0; pt < WS; pt++) {
                const int q = ch * WS + pt, gq = qbase + q;
                cp_async16z(dst0 + (q & (NR - 1)) * C, q <= qmax ? src0 + gq * sst : src0, q <= qmax);
            }
            if (VISC && v < 4) {
                const double *srcf = a.in.FV + v * a.in.vcs + cpv;
                double *dstf = sv + (SV_FV + v) * VS + 2 * (lane & 3);
#pragma unroll
                for (int pt = 0; pt < WS; pt++) {
                    const int q = ch * WS + pt, gq = qbase + q;
                    const bool okf = q <= qmax && gq >= -2 && gq <= nd + 1;
                    cp_async16z(dstf + (q & (NR - 1)) * C, okf ? srcf + gq * vst : srcf, okf);
                }
            }
        }
        cp_async_commit();
    };
    // primitives of chunk `ch` (one point per lane, unconditionally: points past the padded box are
    // stale ring values that only masked lanes read; measured zeta -0.1 ms), from the staged state:
    // prim_calc into registers, prim_store into the ring
    auto prim_calc = [&](int ch, double pv[7]) {
        const int q = ch * WS + ls;
        const double *bq = sv + RG::slot(q, lt);
        const double rho = bq[0], ru = bq[VS], rv = bq[2 * VS], rw = bq[3 * VS], E = bq[4 * VS];
        const double ir = rcp_nr(rho);
        const double u = ru * ir, v = rv * ir, w = rw * ir;
        const double pr = ph.gm1 * fma(-0.5, fma(ru, u, fma(rv, v, rw * w)), E);
        pv[PU] = u;
        pv[PV] = v;
        pv[PW] = w;
        pv[PP] = pr;
        pv[PC] = sqrt_nr(ph.gamma * pr * ir);
        pv[PIS] = rsqrt_nr(rho);
        pv[PH] = (E + pr) * ir;
    };
    auto prim_store = [&](int ch, const double pv[7]) {
        const int q = ch * WS + ls;
        double *bq = sv + RG::slot(q, lt);
#pragma unroll
        for (int k = 0; k < 7; k++) bq[(SV_P + k) * VS] = pv[k];
    };
    auto prims = [&](int ch) {
        double pv[7];
        prim_calc(ch, pv);
        prim_store(ch, pv);
    };

    // prologue: chunks 0 .. LA staged with primitives
    for (int ch = 0; ch <= LA; ch++) issue(ch);
    cp_async_wait_all();
    __syncwarp();
    for (int ch = 0; ch <= LA; ch++) prims(ch);
    __syncwarp();

    // this lane's point at step 0 (interface e = e0-1+ls finishes point e) and its indices
    const int64_t rstep = (D == 0 ? 1 : (D == 1 ? (int64_t)L.n0 : (int64_t)L.n0 * L.n1)) * WS;
    const int64_t pstep = sst * WS;
    int64_t rr, pp;
    {
        const int e = e0 - 1 + ls;
        const int pi = D == 0 ? e : ci, pj = D == 1 ? e : cj, pk = D == 2 ? e : ck;
        rr = (int64_t)pi + (int64_t)L.n0 * (pj + (int64_t)L.n1 * pk);
        pp = at(L, pi, pj, pk);
    }
    double F[5], Fc[5];
#pragma unroll
    for (int c = 0; c < 5; c++) Fc[c] = 0.0;
    for (int st = 0; st < nsteps; st++, rr += rstep, pp += pstep) {
        if (st > 0) {
            // chunk st+LA landed -> primitives (computing the interface setup beside them, as two
            // independent chains, measured 3.5 % slower: register pressure)
            cp_async_wait_all();
            __syncwarp();
            prims(st + LA);
            __syncwarp();
        }
        const int e = e0 - 1 + WS * st + ls;  // this lane's interface e+1/2
        const bool act = lvalid && e <= e1 - 1;
        const bool own = act && e >= e0;      // this lane finishes point e
        const SAcc<NR, C, VISC, RG::CS> A{sv, WS * st + ls + RG::QOFF, lt};  // ring point of stencil point i-2
        // group A: accumulate / update operands of the own point; xi / eta: predicated copies (zero-
        // filled for the other lanes, no branch), zeta: branch (measured: predication there +0.1 ms)
        if constexpr (MODE == 1 || MODE == 4) {
        {
#pragma unroll
            for (int c = 0; c < 5; c++)
                if (c > 0 || MODE != 4) cp_async8z(cb + 32 * c, own ? a.R + c * a.rcs + rr : a.R, own);
            if (MODE == 2 || MODE == 3) {  // J (the zeta sweep finishes the point)
                cp_async8z(cb + 32 * 5, own ? a.in.M + pp : a.in.M, own);
                if (MODE == 3 && a.stage != 0) {
#pragma unroll
                    for (int c = 0; c < 5; c++) cp_async8z(cb + 32 * (6 + c), own ? a.dU + c * L.cs + pp : a.dU, own);
                }
            }
        }
        } else {
        if (own && MODE != 0) {             // group A: accumulate / update operands
#pragma unroll
            for (int c = 0; c < 5; c++)
                if (c > 0 || MODE != 4) cp_async8(cb + 32 * c, a.R + c * a.rcs + rr);
            if (MODE == 2 || MODE == 3) {  // J (the zeta sweep finishes the point)
                cp_async8(cb + 32 * 5, a.in.M + pp);
                if (MODE == 3) {
#pragma unroll
                    for (int c = 0; c < 5; c++) {
                        if (a.stage != 0) cp_async8(cb + 32 * (6 + c), a.dU + c * L.cs + pp);
                    }
                }
            }
        }
        }
        cp_async_commit();
        issue(st + LA + 1);                   // group B: chunk st+LA+1 (slot of chunk st-1)
        {   // every lane evaluates its interface (lanes past the segment end or outside the block on
            // stale ring values) and the inactive lanes' result is masked: no divergent branch around
            // the flux, measured -0.2 ms per 512^3 eta launch
            FluxSetup su;
            if (inv) flux_setup(A, ph, su);
            flux_fields<D, SAcc<NR, C, VISC, RG::CS>, LIM>(A, su, inv, VISC, ph, F);
#pragma unroll
            for (int c = 0; c < 5; c++) F[c] = act ? F[c] : 0.0;
        }
        double dF[5];
        if constexpr (RG::CARRY) {
            // fluxes of step st in slot (st & 1); the left neighbour interface is lane-1 (xi) /
            // lane-8 (eta, zeta) of this step, or the last interface of the line in the last step
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
        asm volatile("cp.async.wait_group 1;\n" ::: "memory");  // group A landed (own data)
        if (own) {
            if (MODE == 0) {
#pragma unroll
                for (int c = 0; c < 5; c++) a.R[c * a.rcs + rr] = dF[c];
            } else {
                double Rt[5];
#pragma unroll
                for (int c = 0; c < 5; c++) Rt[c] = (c == 0 && MODE == 4) ? dF[0] : cb[32 * c] + dF[c];
                if (MODE == 1 || MODE == 4) {
#pragma unroll
                    for (int c = 0; c < 5; c++) a.R[c * a.rcs + rr] = Rt[c];
                } else if (MODE == 2) {
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
                        // U_in of the finished point = stencil point i of the ring (U_in is the
                        // swept state): no second read of U_in
                        a.Uout[c * L.cs + pp] = fma(a.B, du, A.U(2, c));
                    }
                }
            }
        }
        __syncwarp();
    }
    cp_async_wait_all();
}

}  // namespace crocco
