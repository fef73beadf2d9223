// Monte Carlo photon migration with on-demand random numbers
// (§VI, Alg.4 MCPhotonMigration).  C ABI: gg_mc_run
// (include/gg_apps.h).  Compiled with -fmad=false: every fp64 expression is
// evaluated as written (IEEE add/mul/div/sqrt, no contraction), in the same
// order as the CPU oracle's, so the two agree exactly unless a libm log/sin/
// cos result differs by an ulp right at a decision threshold.
//
// One GPU thread per walker; the photon state lives in SoA arrays between
// epochs.  An epoch = one on-demand window of D = 3K draws per walker
// (prng_epoch_begin); every iteration of a thread with work takes exactly
// three prng_next draws at the same program point (so a warp walks the
// expander in lockstep; only the physics diverges) and uses what it needs:
// launch (W0 from draw a), or hop (sleft from a when needed) + boundary
// (Fresnel test with b) or drop + spin (HG cos(theta) from b, psi from c).
// Weights and tallies are int64 fixed point (units 2^-32), so tallies are
// exact integer sums and order independent; the host allreduces them across
// GPUs (NCCL) if sharded.
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <vector>

#include <cuda_runtime.h>

#include "gg_apps.h"
#include "gg_internal.h"
#include "prng.h"
#include "prng_device.cuh"

namespace {

constexpr int kMaxL = GG_MC_MAX_LAYERS;
constexpr int kFixed = 5;  // launched, specular, R_d, T_t, terminated
constexpr double kPi = 3.14159265358979323846;

struct McParams {
    double zb[kMaxL + 1];     // layer boundaries, zb[0] = 0
    double nidx[kMaxL + 2];   // refractive index: 0 = top ambient, nl+1 = bottom ambient
    double mua[kMaxL + 1], mus[kMaxL + 1], g[kMaxL + 1];  // 1-based
    uint64_t qabs[kMaxL + 1]; // round(2^32 mua/mut)
    uint64_t q_sp;            // round(2^32 Rsp)
    uint64_t w_th;            // floor(2^32 w_threshold)
    uint64_t photons_total, threads_total, thread0, threads;
    int nl;
    uint32_t K;               // iterations per epoch (D = 3K)
};

struct McState {
    double *x, *y, *z, *ux, *uy, *uz, *sleft;
    uint64_t *w;
    int32_t *layer;
    uint32_t *alive, *launched;
    uint8_t *busy;   // 1 while the thread still has photons to simulate
};

__device__ __forceinline__ double mc_xi(uint64_t label) {
    return (double)((label >> 11) + 1) * (1.0 / 9007199254740992.0);
}

__device__ __forceinline__ uint64_t mc_frac(uint64_t w, uint64_t q) {
    // (w * q) >> 32 over the full 128-bit product
    return (__umul64hi(w, q) << 32) | ((w * q) >> 32);
}

// Deflection cosine, Henyey-Greenstein phase function (§VI "the angles of
// deflection"; CUDAMCML [1]).  The HG CDF in mu = cos(theta) is
//   F(mu) = (1 - g^2) / (2g) * [(1 + g^2 - 2g mu)^(-1/2) - (1 + g)^(-1)],
// and F(mu) = xi solves to sqrt(1 + g^2 - 2g mu) = (1 - g^2) / (1 + g (2xi - 1)).
__device__ __forceinline__ double hg_cos_theta(double g, double xi) {
    const double t = 2.0 * xi - 1.0;  // isotropic: mu uniform on [-1, 1]
    if (g == 0.0) return t;
    const double k = (1.0 - g * g) / (1.0 + g * t);
    const double mu = (1.0 + g * g - k * k) / (2.0 * g);
    return mu < -1.0 ? -1.0 : (mu > 1.0 ? 1.0 : mu);
}

// Unpolarised Fresnel reflectance from index n1 into n2 at incidence cosine
// c1, as the mean of the squared s- and p-amplitude coefficients
//   r_s = (n1 c1 - n2 c2) / (n1 c1 + n2 c2),  r_p = (n2 c1 - n1 c2) / (n2 c1 + n1 c2),
// c2 = cos of the transmitted angle (Snell, n1 sin t1 = n2 sin t2), written to *c2_out.
// Conventions shared with the oracle's reading (DESIGN R22): within 1e-12 of
// normal incidence c2 = c1; below c1 = 1e-6 (grazing) and beyond the critical
// angle the photon is reflected (R = 1, c2 = 0).
__device__ __forceinline__ double fresnel_unpolarised(double n1, double n2, double c1,
                                                      double *c2_out) {
    if (n1 == n2) {
        *c2_out = c1;
        return 0.0;
    }
    double c2;
    if (c1 > 1.0 - 1.0e-12) {
        c2 = c1;
    } else if (c1 < 1.0e-6) {
        *c2_out = 0.0;
        return 1.0;
    } else {
        const double s2 = n1 * sqrt(1.0 - c1 * c1) / n2;
        if (s2 >= 1.0) {
            *c2_out = 0.0;
            return 1.0;
        }
        c2 = sqrt(1.0 - s2 * s2);
    }
    *c2_out = c2;
    const double rs = (n1 * c1 - n2 * c2) / (n1 * c1 + n2 * c2);
    const double rp = (n2 * c1 - n1 * c2) / (n2 * c1 + n1 * c2);
    return 0.5 * (rs * rs + rp * rp);
}

// Scattering: rotate the unit direction u by the polar angle theta (cos =
// cost) and the azimuth psi about u, in the orthonormal frame
//   e1 = (ux uz, uy uz, -(1 - uz^2)) / sqrt(1 - uz^2),  e2 = (-uy, ux, 0) / sqrt(1 - uz^2):
//   u' = cost u + sint (cos psi e1 + sin psi e2).
// Near the poles (|uz| > 0.99999) the frame is (x, y, sign(uz) z).
__device__ __forceinline__ void scatter_direction(double cost, double psi, double &ux, double &uy,
                                                  double &uz) {
    const double sint = sqrt(1.0 - cost * cost);
    double sp, cp;
    sincos(psi, &sp, &cp);
    if (fabs(uz) > 0.99999) {
        ux = sint * cp;
        uy = sint * sp;
        uz = uz >= 0.0 ? cost : -cost;
        return;
    }
    const double rho = sqrt(1.0 - uz * uz);
    const double sr = sint / rho;  // one division for both frame weights
    const double a = sr * cp, b = sr * sp;  // weights of rho*e1, rho*e2
    const double nx = ux * cost + (a * ux * uz - b * uy);
    const double ny = uy * cost + (a * uy * uz + b * ux);
    const double nz = uz * cost - sint * cp * rho;
    ux = nx;
    uy = ny;
    uz = nz;
}

__global__ void mc_init_state(McState s, uint64_t n) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    s.alive[i] = 0;
    s.launched[i] = 0;
    s.w[i] = 0;
    // geometry of a thread without a photon is never used before launch sets
    // it, but the epoch kernel loads it unconditionally: define it (initcheck)
    s.x[i] = s.y[i] = s.z[i] = 0.0;
    s.ux[i] = s.uy[i] = 0.0;
    s.uz[i] = 1.0;
    s.sleft[i] = 0.0;
    s.layer[i] = 0;
    s.busy[i] = 1;
}

// MODE: PRNG_WALK_L64 for the paper's generator (only that walk compiled into
// the epoch loop), PRNG_WALK_AUTO (run-time dispatch) for other parameters.
template <int MINB, int MODE>
__global__ void __launch_bounds__(128, MINB) mc_epoch(const __grid_constant__ prng_view v,
                                                      McParams P, McState S,
                                                unsigned long long *tallies,
                                                long long *per_thread,
                                                unsigned long long *counters) {
    // the paper's generator (PRNG_WALK_L64): composed-step table in shared memory
    constexpr bool TAB = MODE == PRNG_WALK_L64;
    __shared__ __align__(PRNG_TABLE_ALIGN) uint32_t tab[TAB ? PRNG_TABLE_WORDS : 4];
    if (TAB) prng_table_stage(&v, tab);  // made visible by the __syncthreads below
    const uint64_t slot = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int nt = kFixed + P.nl;
    // block tallies in shared memory (int64 atomics: exact, order independent)
    __shared__ unsigned long long s_tal[kFixed + kMaxL];
    for (int k = threadIdx.x; k < kFixed + kMaxL; k += blockDim.x) s_tal[k] = 0;
    __syncthreads();
    long long *my_row = nullptr;
    auto tally = [&](int k, uint64_t v) {
        if (v) atomicAdd(&s_tal[k], (unsigned long long)v);
        if (my_row) my_row[k] += (long long)v;
    };
    unsigned long long launched_now = 0, interactions = 0, draws = 0, done = 0;
    if (slot < v.Wv) {
        // the window holds the threads that still had work one epoch ago
        const uint64_t i = v.wmap ? v.wmap[slot] : slot;
        const uint64_t tg = P.thread0 + i;
        if (per_thread) my_row = per_thread + i * nt;
        const uint64_t budget =
            P.photons_total / P.threads_total + (tg < P.photons_total % P.threads_total ? 1 : 0);
        double x = S.x[i], y = S.y[i], z = S.z[i], ux = S.ux[i], uy = S.uy[i], uz = S.uz[i];
        double sleft = S.sleft[i];
        uint64_t w = S.w[i];
        int layer = S.layer[i];
        bool alive = S.alive[i] != 0;
        uint32_t launched = S.launched[i];
        prng_state st = prng_state_load(&v, (uint32_t)slot);
        for (uint32_t it = 0; it < P.K; it++) {
            if (!alive && launched == budget) break;
            // three draws at a convergent point (R22), their loads in flight
            // together; the table walk's three copies unrolled (the rolled
            // form kept the R2P walk inside the instruction cache; the table
            // walk is shorter: 108.8 -> 104.2 ms of C4 kernel time unrolled)
            uint64_t d3[3];
            if (TAB)
                prng_next_n_table<3, false>(&st, &v, tab, d3);
            else
                prng_next_n<3, true, MODE>(&st, &v, d3);
            const uint64_t la = d3[0], lb = d3[1], lc = d3[2];
            draws += 3;
            if (!alive) {
                // Alg.4 l.3: launch a photon with its weight from getnextrand()
                const uint64_t w0 = (la >> 32) + 1;
                const uint64_t sp = mc_frac(w0, P.q_sp);
                tally(0, w0);
                tally(1, sp);
                w = w0 - sp;
                x = 0.0;
                y = 0.0;
                z = 0.0;
                ux = 0.0;
                uy = 0.0;
                uz = 1.0;
                sleft = 0.0;
                layer = 1;
                alive = true;
                launched++;
                launched_now++;
                continue;
            }
            const double mua = P.mua[layer], mus = P.mus[layer], g = P.g[layer];
            const double mut = mua + mus;
            if (sleft == 0.0) sleft = -log(mc_xi(la));
            double db;
            if (uz > 0.0)
                db = (P.zb[layer] - z) / uz;
            else if (uz < 0.0)
                db = (P.zb[layer - 1] - z) / uz;
            else
                db = INFINITY;
            const double s = sleft / mut;
            if (s > db) {
                x = x + db * ux;
                y = y + db * uy;
                z = z + db * uz;
                sleft = sleft - db * mut;
                const int nb = uz < 0.0 ? layer - 1 : layer + 1;
                const double n1 = P.nidx[layer], n2 = P.nidx[nb];
                double ca2;
                const double r = fresnel_unpolarised(n1, n2, fabs(uz), &ca2);
                bool reflect = false;
                if (n1 != n2) reflect = mc_xi(lb) <= r;
                if (reflect) {
                    uz = -uz;
                } else if (nb == 0 || nb == P.nl + 1) {
                    tally(nb == 0 ? 2 : 3, w);
                    w = 0;
                    alive = false;
                } else {
                    layer = nb;
                    if (n1 != n2) {  // Snell: tangential part scales by n1/n2, |uz| = cos t2
                        const double eta = n1 / n2;
                        ux *= eta;
                        uy *= eta;
                        uz = copysign(ca2, uz);
                    }
                }
            } else {
                x = x + s * ux;
                y = y + s * uy;
                z = z + s * uz;
                sleft = 0.0;
                const uint64_t dw = mc_frac(w, P.qabs[layer]);
                w -= dw;
                tally(kFixed + layer - 1, dw);
                scatter_direction(hg_cos_theta(g, mc_xi(lb)), 2.0 * kPi * mc_xi(lc), ux, uy, uz);
                interactions++;
                if (w < P.w_th) {
                    tally(4, w);
                    w = 0;
                    alive = false;
                }
            }
        }
        prng_state_store(&v, &st);
        S.x[i] = x;
        S.y[i] = y;
        S.z[i] = z;
        S.ux[i] = ux;
        S.uy[i] = uy;
        S.uz[i] = uz;
        S.sleft[i] = sleft;
        S.w[i] = w;
        S.layer[i] = layer;
        S.alive[i] = alive ? 1u : 0u;
        S.launched[i] = launched;
        done = (!alive && launched == budget) ? 1 : 0;
        S.busy[i] = done ? 0 : 1;
    }
    __syncthreads();
    for (int k = threadIdx.x; k < nt; k += blockDim.x)
        if (s_tal[k]) atomicAdd(&tallies[k], s_tal[k]);
    const unsigned full = 0xFFFFFFFFu;
    unsigned long long c[4] = {launched_now, draws, interactions, done};
    for (int k = 0; k < 4; k++) {
        unsigned long long vsum = c[k];
        for (int o = 16; o > 0; o >>= 1) vsum += __shfl_down_sync(full, vsum, o);
        if ((threadIdx.x & 31) == 0 && vsum) atomicAdd(&counters[k], vsum);
    }
}

// GG_MC_MINB hook: blocks per SM in the register budget (default 8).
template <int MODE>
void launch_epoch(int minb, unsigned grid, cudaStream_t s, const prng_view &v, const McParams &P,
                  const McState &S, unsigned long long *tal, long long *per_thread,
                  unsigned long long *cnt) {
    if (minb >= 12)
        mc_epoch<12, MODE><<<grid, 128, 0, s>>>(v, P, S, tal, per_thread, cnt);
    else if (minb >= 8)
        mc_epoch<8, MODE><<<grid, 128, 0, s>>>(v, P, S, tal, per_thread, cnt);
    else if (minb >= 6)
        mc_epoch<6, MODE><<<grid, 128, 0, s>>>(v, P, S, tal, per_thread, cnt);
    else
        mc_epoch<4, MODE><<<grid, 128, 0, s>>>(v, P, S, tal, per_thread, cnt);
}

struct Fail {
    int rc;
};
#define MCK(call)                                              \
    do {                                                       \
        cudaError_t _e = (call);                               \
        if (_e != cudaSuccess) throw Fail{PRNG_E_CUDA};        \
    } while (0)
#define MRC(call)                                              \
    do {                                                       \
        int _r = (call);                                       \
        if (_r != PRNG_OK) throw Fail{_r};                     \
    } while (0)

uint64_t q32(double f) { return (uint64_t)llround(ldexp(f, 32)); }

}  // namespace

extern "C" int gg_mc_run(prng_t *h, const gg_mc_config *cfg, int64_t *tallies, int64_t *per_thread,
                         int64_t *stats, void *stream) {
    if (!h || !cfg || !tallies || !cfg->layers) return PRNG_E_INVALID;
    if (cfg->nlayers < 1 || cfg->nlayers > kMaxL || cfg->threads == 0 ||
        cfg->threads_total == 0 || cfg->epoch_draws < 3 || cfg->epoch_draws % 3 != 0 ||
        cfg->thread0 + cfg->threads > cfg->threads_total)
        return PRNG_E_INVALID;
    if (per_thread && ((uintptr_t)per_thread % 8) != 0) return PRNG_E_INVALID;
    cudaStream_t s = (cudaStream_t)stream;
    McParams P{};
    P.nl = cfg->nlayers;
    P.zb[0] = 0.0;
    P.nidx[0] = cfg->n_top;
    for (int l = 1; l <= P.nl; l++) {
        const gg_mc_layer &L = cfg->layers[l - 1];
        if (!(L.d > 0.0) || L.mua < 0.0 || L.mus < 0.0 || !(L.mua + L.mus > 0.0) || L.g <= -1.0 ||
            L.g >= 1.0)
            return PRNG_E_INVALID;
        P.zb[l] = P.zb[l - 1] + L.d;
        P.nidx[l] = L.n;
        P.mua[l] = L.mua;
        P.mus[l] = L.mus;
        P.g[l] = L.g;
        P.qabs[l] = q32(L.mua / (L.mua + L.mus));
    }
    P.nidx[P.nl + 1] = cfg->n_bottom;
    double rsp = (cfg->n_top - P.nidx[1]) / (cfg->n_top + P.nidx[1]);
    rsp = rsp * rsp;
    P.q_sp = q32(rsp);
    P.w_th = (uint64_t)floor(ldexp(cfg->w_threshold, 32));
    P.photons_total = cfg->photons_total;
    P.threads_total = cfg->threads_total;
    P.thread0 = cfg->thread0;
    P.threads = cfg->threads;
    P.K = cfg->epoch_draws / 3;
    const int nt = kFixed + P.nl;

    std::vector<void *> bufs;
    cudaMemPool_t pool = gg::scratch_pool();
    if (!pool) return PRNG_E_CUDA;
    auto alloc = [&](size_t bytes) -> void * {
        void *p = nullptr;
        MCK(cudaMallocFromPoolAsync(&p, bytes, pool, s));
        bufs.push_back(p);
        return p;
    };
    int rc = PRNG_OK;
    try {
        const uint64_t n = cfg->threads;
        McState S;
        S.x = (double *)alloc(n * 8);
        S.y = (double *)alloc(n * 8);
        S.z = (double *)alloc(n * 8);
        S.ux = (double *)alloc(n * 8);
        S.uy = (double *)alloc(n * 8);
        S.uz = (double *)alloc(n * 8);
        S.sleft = (double *)alloc(n * 8);
        S.w = (uint64_t *)alloc(n * 8);
        S.layer = (int32_t *)alloc(n * 4);
        S.alive = (uint32_t *)alloc(n * 4);
        S.launched = (uint32_t *)alloc(n * 4);
        S.busy = (uint8_t *)alloc(n);
        uint32_t *d_list = (uint32_t *)alloc(n * 4);
        int32_t *d_count = (int32_t *)alloc(8);
        void *sel_tmp = alloc(gg::compact_scratch_bytes((int64_t)n));
        unsigned long long *d_tal = (unsigned long long *)alloc(nt * 8);
        unsigned long long *d_cnt = (unsigned long long *)alloc(4 * 8);
        MCK(cudaMemsetAsync(d_tal, 0, nt * 8, s));
        MCK(cudaMemsetAsync(d_cnt, 0, 4 * 8, s));
        if (per_thread) MCK(cudaMemsetAsync(per_thread, 0, n * nt * 8, s));
        mc_init_state<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(S, n);
        cudaEvent_t e0, e1;
        MCK(cudaEventCreate(&e0));
        MCK(cudaEventCreate(&e1));
        MCK(cudaEventRecord(e0, s));
        // pinned host buffers: counters, active count and active list (the D2H
        // reads must not block the host FEED of the next window)
        unsigned long long *counters = nullptr;
        uint32_t *h_list = nullptr;
        MCK(cudaMallocHost(&counters, 4 * sizeof(unsigned long long) + 8));
        MCK(cudaMallocHost(&h_list, n * 4));
        int32_t *h_count = (int32_t *)(counters + 4);
        std::vector<uint32_t> feed_list;  // walkers of the next window (one epoch of lag)
        int64_t epochs = 0;
        double kernel_ms = 0.0;
        uint64_t window_slots = 0;
        cudaEvent_t k0, k1, kc;
        MCK(cudaEventCreate(&k0));
        MCK(cudaEventCreate(&k1));
        MCK(cudaEventCreateWithFlags(&kc, cudaEventDisableTiming));
        try {
            MRC(prng_epoch_reserve(h, n, cfg->epoch_draws));  // no allocation inside the loop
            MRC(prng_epoch_begin(h, n, cfg->epoch_draws, s));
            uint64_t wslots = n;
            for (;;) {
                prng_view v;
                MRC(prng_device_view(h, &v, sizeof(v)));
                MCK(cudaEventRecord(k0, s));
                static const int minb = getenv("GG_MC_MINB") ? atoi(getenv("GG_MC_MINB")) : 8;
                const unsigned grid = (unsigned)((wslots + 127) / 128);
                if (prng_walk_mode(&v) == PRNG_WALK_L64)
                    launch_epoch<PRNG_WALK_L64>(minb, grid, s, v, P, S, d_tal,
                                                (long long *)per_thread, d_cnt);
                else
                    launch_epoch<PRNG_WALK_AUTO>(minb, grid, s, v, P, S, d_tal,
                                                 (long long *)per_thread, d_cnt);
                MCK(cudaGetLastError());
                MCK(cudaEventRecord(k1, s));
                MRC(prng_epoch_end(h, s));
                epochs++;
                window_slots += wslots;
                // threads that still have work after this epoch
                MCK(gg::compact_flagged(nullptr, S.busy, (int64_t)n, (int32_t *)d_list, nullptr, d_count,
                                        nullptr, 0, sel_tmp, s));
                MCK(cudaMemcpyAsync(h_count, d_count, 4, cudaMemcpyDeviceToHost, s));
                MCK(cudaMemcpyAsync(h_list, d_list, n * 4, cudaMemcpyDeviceToHost, s));
                MCK(cudaMemcpyAsync(counters, d_cnt, 4 * sizeof(unsigned long long),
                                    cudaMemcpyDeviceToHost, s));
                MCK(cudaEventRecord(kc, s));
                // FEED + TRANSFER of the next window overlap this epoch's kernel
                // (Alg.4 l.7: "Generate and transfer new bin in an overlapping
                // manner").  Its walkers are the threads known to be busy one
                // epoch ago (a superset of those busy now); a thread that has
                // finished in between simply does not draw.
                if (epochs == 1) {
                    MRC(prng_epoch_begin(h, n, cfg->epoch_draws, s));
                    wslots = n;
                } else {
                    MRC(prng_epoch_begin_list(h, feed_list.data(), feed_list.size(),
                                              cfg->epoch_draws, s));
                    wslots = feed_list.size();
                }
                MCK(cudaEventSynchronize(kc));
                float ms = 0.0f;
                MCK(cudaEventElapsedTime(&ms, k0, k1));
                kernel_ms += ms;
                if (*h_count == 0) {
                    MRC(prng_epoch_end(h, s));  // discard the speculative window
                    break;
                }
                feed_list.assign(h_list, h_list + *h_count);
            }
        } catch (const Fail &) {
            cudaFreeHost(counters);
            cudaFreeHost(h_list);
            throw;
        }
        const unsigned long long c_launched = counters[0], c_draws = counters[1],
                                 c_inter = counters[2];
        cudaFreeHost(counters);
        cudaFreeHost(h_list);
        MCK(cudaEventRecord(e1, s));
        std::vector<unsigned long long> ht(nt);
        MCK(cudaMemcpyAsync(ht.data(), d_tal, nt * 8, cudaMemcpyDeviceToHost, s));
        MCK(cudaStreamSynchronize(s));
        for (int k = 0; k < nt; k++) tallies[k] += (int64_t)ht[k];
        if (stats) {
            float total_ms = 0.0f;
            MCK(cudaEventElapsedTime(&total_ms, e0, e1));
            stats[0] = (int64_t)c_launched;    // photons launched
            stats[1] = (int64_t)c_draws;       // draws taken by the physics
            stats[2] = epochs;
            stats[3] = (int64_t)c_inter;       // interactions
            stats[4] = (int64_t)(kernel_ms * 1000.0);  // microseconds in mc_epoch kernels
            stats[5] = (int64_t)(total_ms * 1000.0);   // microseconds end to end (feed incl.)
            stats[6] = (int64_t)window_slots;          // walker-epochs fed (x D draws of bits)
        }
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
        cudaEventDestroy(k0);
        cudaEventDestroy(k1);
        cudaEventDestroy(kc);
    } catch (const Fail &f) {
        rc = f.rc;
    }
    for (void *p : bufs) cudaFreeAsync(p, s);
    if (cudaStreamSynchronize(s) != cudaSuccess && rc == PRNG_OK) rc = PRNG_E_CUDA;
    return rc;
}
