// libbarracuda C ABI (include/barracuda.h): argument validation and dispatch.
#include <cuda_runtime.h>

#include <cstdlib>
#include <atomic>
#include <mutex>

#include "common.cuh"

namespace bc {

int run_sumfact3d(int64_t, int, const double*, const double*, const double*, const double*, double*, double*,
                  cudaStream_t);
int run_sumfact3d_f32(int64_t, int, const float*, const float*, const float*, const float*, float*, cudaStream_t);
int run_sumfact2d(int64_t, int, const double*, const double*, const double*, double*, cudaStream_t);
int run_local_grad3(int64_t, int, const double*, const double*, double*, double*, double*, cudaStream_t);
int run_local_grad3_t(int64_t, int, const double*, const double*, const double*, const double*, double*, cudaStream_t);
int run_ax_e(int64_t, int, const double*, const double*, const double*, double*, cudaStream_t);
int run_ccsdt(int fam, const int* ext7, double* t3, const int* vs, int nv, const double* const* opA,
              const double* const* opB, cudaStream_t s, const double* eps_h = nullptr, const double* eps_p = nullptr,
              double* ws = nullptr);
int run_sumfact3d_mma(int64_t, int, const double*, const double*, const double*, const double*, double*, double*,
                      cudaStream_t);
int run_sumfact2d_mma(int64_t, int, const double*, const double*, const double*, double*, cudaStream_t);
int run_local_grad3_mma(int64_t, int, const double*, const double*, double*, double*, double*, cudaStream_t);
int run_ccsdt_triples_energy(const int* ext7, const double* const* t1, const double* const* v2s1,
                             const double* const* t2d1, const double* const* v2d1, const double* const* t2d2,
                             const double* const* v2d2, const double* eps_h, const double* eps_p, double* ws,
                             cudaStream_t s);
int run_sumsq(int64_t n, const double* x, double* ws, cudaStream_t s);
int run_probe_fp64(int kind, int iters, double* scratch, double* flops, cudaStream_t s);
int probe_scratch_doubles();
int run_energy(const int* ext7, const double* t3, const double* eh, const double* ep, double* ws, cudaStream_t s);
template <typename T>
int run_fill(int kind, uint64_t seed, uint64_t tid, uint64_t offset, int64_t n, double lo, double hi, T* out,
             cudaStream_t s);

// Tensor-core (DMMA) spectral kernels are used where they cover p (spectral_mma.cu); the
// environment variable BC_SPECTRAL_PATH=dfma forces the DFMA kernels (A/B measurements).
static bool spectral_mma_enabled() {
    static const bool on = [] {
        const char* v = getenv("BC_SPECTRAL_PATH");
        return !(v && v[0] == 'd');
    }();
    return on;
}

static thread_local int g_last_cuda_error = 0;
static thread_local int64_t g_launches = 0;
void set_last_cuda_error(cudaError_t e) { g_last_cuda_error = (int)e; }
void count_launch(int n) { g_launches += n; }

int current_device() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= BC_MAX_DEVICES) dev = 0;
    return dev;
}

int num_sms() {
    static std::atomic<int> sms[BC_MAX_DEVICES];
    const int dev = current_device();
    int v = sms[dev].load(std::memory_order_relaxed);
    if (v == 0) {
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) v = 148;
        sms[dev].store(v, std::memory_order_relaxed);
    }
    return v;
}

// ---------------------------------------------------------------- validation helpers
static bool aligned(const void* p, int a) { return (reinterpret_cast<uintptr_t>(p) % a) == 0; }
static bool overlap(const void* a, size_t na, const void* b, size_t nb) {
    const uintptr_t x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
    return na && nb && x < y + nb && y < x + na;
}

#define BC_REQUIRE(cond, code) \
    do {                       \
        if (!(cond)) return (code); \
    } while (0)

static int check_spectral(int64_t N, int p) {
    BC_REQUIRE(N >= 0, BC_ERR_ARG);
    BC_REQUIRE(p >= 1, BC_ERR_ARG);
    BC_REQUIRE(p <= BC_MAX_P, BC_ERR_UNSUPPORTED);
    return BC_OK;
}

static int check_dims(const bc_tile_dims* d, bool needk) {
    BC_REQUIRE(d != nullptr, BC_ERR_ARG);
    const int e[7] = {d->h1, d->h2, d->h3, d->p4, d->p5, d->p6, d->k};
    for (int q = 0; q < (needk ? 7 : 6); ++q) {
        BC_REQUIRE(e[q] > 0, BC_ERR_ARG);
        BC_REQUIRE(e[q] <= BC_MAX_TILE_EXTENT, BC_ERR_UNSUPPORTED);
    }
    return BC_OK;
}

static void dims_to_ext(const bc_tile_dims* d, int* e, bool needk) {
    e[0] = d->h1; e[1] = d->h2; e[2] = d->h3; e[3] = d->p4; e[4] = d->p5; e[5] = d->p6;
    e[6] = needk ? d->k : 1;
}

static size_t t3_elems(const int* e) { return (size_t)e[0] * e[1] * e[2] * e[3] * e[4] * e[5]; }

// family: 1 = d1, 2 = d2, 3 = s1
static void operand_elems(int fam, const int* e, size_t* na, size_t* nb) {
    if (fam == 1) { *na = (size_t)e[6] * e[3] * e[4] * e[0]; *nb = (size_t)e[2] * e[1] * e[5] * e[6]; }
    else if (fam == 2) { *na = (size_t)e[6] * e[3] * e[0] * e[1]; *nb = (size_t)e[6] * e[2] * e[5] * e[4]; }
    else { *na = (size_t)e[3] * e[0]; *nb = (size_t)e[2] * e[1] * e[5] * e[4]; }
}

static int ccsdt_one(int fam, int variant, const bc_tile_dims* d, double* t3, const double* a,
                     const double* b, void* stream) {
    const bool needk = fam != 3;
    int st = check_dims(d, needk);
    if (st) return st;
    BC_REQUIRE(variant >= 1 && variant <= 9, BC_ERR_ARG);
    BC_REQUIRE(t3 && a && b, BC_ERR_ARG);
    BC_REQUIRE(aligned(t3, 16) && aligned(a, 16) && aligned(b, 16), BC_ERR_ALIGN);
    int e[7];
    dims_to_ext(d, e, needk);
    size_t na, nb;
    operand_elems(fam, e, &na, &nb);
    const size_t n3 = t3_elems(e);
    BC_REQUIRE(!overlap(t3, n3 * 8, a, na * 8) && !overlap(t3, n3 * 8, b, nb * 8), BC_ERR_ALIAS);
    return run_ccsdt(fam, e, t3, &variant, 1, &a, &b, as_stream(stream));
}

// eps_h/eps_p/ws non-null: also ws[0] = energy check of the updated t3 (bc_check_energy)
static int ccsdt_fused(int fam, const bc_tile_dims* d, double* t3, const double* const* A,
                       const double* const* B, void* stream, const double* eps_h = nullptr,
                       const double* eps_p = nullptr, double* ws = nullptr) {
    const bool needk = fam != 3;
    int st = check_dims(d, needk);
    if (st) return st;
    BC_REQUIRE(t3 && A && B, BC_ERR_ARG);
    BC_REQUIRE(aligned(t3, 16), BC_ERR_ALIGN);
    int e[7];
    dims_to_ext(d, e, needk);
    size_t na, nb;
    operand_elems(fam, e, &na, &nb);
    const size_t n3 = t3_elems(e);
    if (ws) {
        BC_REQUIRE(eps_h && eps_p, BC_ERR_ARG);
        BC_REQUIRE(aligned(eps_h, 8) && aligned(eps_p, 8) && aligned(ws, 8), BC_ERR_ALIGN);
        BC_REQUIRE(!overlap(ws, BC_CHECK_WS_DOUBLES * 8, t3, n3 * 8), BC_ERR_ALIAS);
    }
    int vs[9], nv = 0;
    const double* pa[9];
    const double* pb[9];
    for (int v = 1; v <= 9; ++v) {
        if (!A[v - 1]) continue;
        BC_REQUIRE(B[v - 1] != nullptr, BC_ERR_ARG);
        BC_REQUIRE(aligned(A[v - 1], 16) && aligned(B[v - 1], 16), BC_ERR_ALIGN);
        BC_REQUIRE(!overlap(t3, n3 * 8, A[v - 1], na * 8) && !overlap(t3, n3 * 8, B[v - 1], nb * 8), BC_ERR_ALIAS);
        vs[nv] = v;
        pa[nv] = A[v - 1];
        pb[nv] = B[v - 1];
        ++nv;
    }
    if (nv == 0) return ws ? run_energy(e, t3, eps_h, eps_p, ws, as_stream(stream)) : BC_OK;
    const bool same_geometry = (e[0] == e[1] && e[1] == e[2] && e[3] == e[4] && e[4] == e[5]);
    if (same_geometry) return run_ccsdt(fam, e, t3, vs, nv, pa, pb, as_stream(stream), eps_h, eps_p, ws);
    for (int t = 0; t < nv; ++t) {  // variants' t3 geometries differ: ascending single-variant passes
        st = run_ccsdt(fam, e, t3, &vs[t], 1, &pa[t], &pb[t], as_stream(stream));
        if (st) return st;
    }
    if (ws) return run_energy(e, t3, eps_h, eps_p, ws, as_stream(stream));
    return BC_OK;
}

static int sumfact3d_impl(int64_t N, int p, const double* A, const double* B, const double* C, const double* U,
                          double* V, double* ws, void* stream) {
    int st = check_spectral(N, p);
    if (st) return st;
    BC_REQUIRE(ws == nullptr || aligned(ws, 8), BC_ERR_ALIGN);
    if (N == 0) {
        if (ws) return run_sumsq(0, V, ws, as_stream(stream));  // ws[0] = 0
        return BC_OK;
    }
    BC_REQUIRE(A && B && C && U && V, BC_ERR_ARG);
    BC_REQUIRE(aligned(A, 16) && aligned(B, 16) && aligned(C, 16) && aligned(U, 16) && aligned(V, 16), BC_ERR_ALIGN);
    const size_t nb = (size_t)N * (p + 1) * (p + 1) * (p + 1) * 8, ob = (size_t)(p + 1) * (p + 1) * 8;
    BC_REQUIRE(!overlap(V, nb, U, nb) && !overlap(V, nb, A, ob) && !overlap(V, nb, B, ob) && !overlap(V, nb, C, ob),
               BC_ERR_ALIAS);
    BC_REQUIRE(!ws || (!overlap(ws, BC_CHECK_WS_DOUBLES * 8, V, nb) && !overlap(ws, BC_CHECK_WS_DOUBLES * 8, U, nb)),
               BC_ERR_ALIAS);
    if (spectral_mma_enabled()) {
        const int st2 = run_sumfact3d_mma(N, p, A, B, C, U, V, ws, as_stream(stream));
        if (st2 != 1) return st2;  // 1: p not covered by the tensor-core kernels
    }
    return run_sumfact3d(N, p, A, B, C, U, V, ws, as_stream(stream));
}

}  // namespace bc

using namespace bc;

extern "C" {

int bc_sumfact3d(int64_t N, int p, const double* A, const double* B, const double* C, const double* U,
                 double* V, void* stream) {
    return sumfact3d_impl(N, p, A, B, C, U, V, nullptr, stream);
}

int bc_sumfact3d_check(int64_t N, int p, const double* A, const double* B, const double* C, const double* U,
                       double* V, double* ws, void* stream) {
    BC_REQUIRE(ws != nullptr, BC_ERR_ARG);
    return sumfact3d_impl(N, p, A, B, C, U, V, ws, stream);
}

int bc_sumfact3d_f32(int64_t N, int p, const float* A, const float* B, const float* C, const float* U, float* V,
                     void* stream) {
    int st = check_spectral(N, p);
    if (st || N == 0) return st;
    BC_REQUIRE(A && B && C && U && V, BC_ERR_ARG);
    BC_REQUIRE(aligned(A, 8) && aligned(B, 8) && aligned(C, 8) && aligned(U, 16) && aligned(V, 16), BC_ERR_ALIGN);
    const size_t nb = (size_t)N * (p + 1) * (p + 1) * (p + 1) * 4, ob = (size_t)(p + 1) * (p + 1) * 4;
    BC_REQUIRE(!overlap(V, nb, U, nb) && !overlap(V, nb, A, ob) && !overlap(V, nb, B, ob) && !overlap(V, nb, C, ob),
               BC_ERR_ALIAS);
    return run_sumfact3d_f32(N, p, A, B, C, U, V, as_stream(stream));
}

int bc_sumfact2d(int64_t N, int p, const double* A, const double* B, const double* U, double* V, void* stream) {
    int st = check_spectral(N, p);
    if (st || N == 0) return st;
    BC_REQUIRE(A && B && U && V, BC_ERR_ARG);
    BC_REQUIRE(aligned(A, 16) && aligned(B, 16) && aligned(U, 16) && aligned(V, 16), BC_ERR_ALIGN);
    const size_t nb = (size_t)N * (p + 1) * (p + 1) * 8, ob = (size_t)(p + 1) * (p + 1) * 8;
    BC_REQUIRE(!overlap(V, nb, U, nb) && !overlap(V, nb, A, ob) && !overlap(V, nb, B, ob), BC_ERR_ALIAS);
    if (spectral_mma_enabled()) {
        const int st2 = run_sumfact2d_mma(N, p, A, B, U, V, as_stream(stream));
        if (st2 != 1) return st2;  // 1: p not covered by the tensor-core kernels
    }
    return run_sumfact2d(N, p, A, B, U, V, as_stream(stream));
}

int bc_local_grad3(int64_t N, int p, const double* D, const double* U, double* ur, double* us, double* ut,
                   void* stream) {
    int st = check_spectral(N, p);
    if (st || N == 0) return st;
    BC_REQUIRE(D && U && ur && us && ut, BC_ERR_ARG);
    BC_REQUIRE(aligned(D, 16) && aligned(U, 16) && aligned(ur, 16) && aligned(us, 16) && aligned(ut, 16), BC_ERR_ALIGN);
    const size_t nb = (size_t)N * (p + 1) * (p + 1) * (p + 1) * 8, ob = (size_t)(p + 1) * (p + 1) * 8;
    double* outs[3] = {ur, us, ut};
    for (int i = 0; i < 3; ++i) {
        BC_REQUIRE(!overlap(outs[i], nb, U, nb) && !overlap(outs[i], nb, D, ob), BC_ERR_ALIAS);
        for (int j = i + 1; j < 3; ++j) BC_REQUIRE(!overlap(outs[i], nb, outs[j], nb), BC_ERR_ALIAS);
    }
    if (spectral_mma_enabled()) {
        const int st2 = run_local_grad3_mma(N, p, D, U, ur, us, ut, as_stream(stream));
        if (st2 != 1) return st2;  // 1: p not covered by the tensor-core kernels
    }
    return run_local_grad3(N, p, D, U, ur, us, ut, as_stream(stream));
}

int bc_local_grad3_t(int64_t N, int p, const double* D, const double* ur, const double* us, const double* ut,
                     double* U, void* stream) {
    int st = check_spectral(N, p);
    if (st || N == 0) return st;
    BC_REQUIRE(D && U && ur && us && ut, BC_ERR_ARG);
    BC_REQUIRE(aligned(D, 16) && aligned(U, 16) && aligned(ur, 16) && aligned(us, 16) && aligned(ut, 16), BC_ERR_ALIGN);
    const size_t nb = (size_t)N * (p + 1) * (p + 1) * (p + 1) * 8, ob = (size_t)(p + 1) * (p + 1) * 8;
    BC_REQUIRE(!overlap(U, nb, ur, nb) && !overlap(U, nb, us, nb) && !overlap(U, nb, ut, nb) && !overlap(U, nb, D, ob),
               BC_ERR_ALIAS);
    return run_local_grad3_t(N, p, D, ur, us, ut, U, as_stream(stream));
}

int bc_ax_e(int64_t N, int p, const double* D, const double* U, const double* G, double* W, void* stream) {
    int st = check_spectral(N, p);
    if (st || N == 0) return st;
    BC_REQUIRE(D && U && G && W, BC_ERR_ARG);
    BC_REQUIRE(aligned(D, 16) && aligned(U, 16) && aligned(G, 16) && aligned(W, 16), BC_ERR_ALIGN);
    const size_t nb = (size_t)N * (p + 1) * (p + 1) * (p + 1) * 8, ob = (size_t)(p + 1) * (p + 1) * 8;
    BC_REQUIRE(!overlap(W, nb, U, nb) && !overlap(W, nb, G, 6 * nb) && !overlap(W, nb, D, ob), BC_ERR_ALIAS);
    return run_ax_e(N, p, D, U, G, W, as_stream(stream));
}

int bc_ccsdt_d1(int variant, const bc_tile_dims* d, double* t3, const double* t2, const double* v2, void* stream) {
    return ccsdt_one(1, variant, d, t3, t2, v2, stream);
}
int bc_ccsdt_d2(int variant, const bc_tile_dims* d, double* t3, const double* t2, const double* v2, void* stream) {
    return ccsdt_one(2, variant, d, t3, t2, v2, stream);
}
int bc_ccsdt_s1(int variant, const bc_tile_dims* d, double* t3, const double* t1, const double* v2, void* stream) {
    return ccsdt_one(3, variant, d, t3, t1, v2, stream);
}
int bc_ccsdt_d1_fused(const bc_tile_dims* d, double* t3, const double* const t2[9], const double* const v2[9],
                      void* stream) {
    return ccsdt_fused(1, d, t3, t2, v2, stream);
}
int bc_ccsdt_d2_fused(const bc_tile_dims* d, double* t3, const double* const t2[9], const double* const v2[9],
                      void* stream) {
    return ccsdt_fused(2, d, t3, t2, v2, stream);
}
int bc_ccsdt_fused_energy(int family, const bc_tile_dims* d, double* t3, const double* const a[9],
                          const double* const b[9], const double* eps_h, const double* eps_p, double* ws,
                          void* stream) {
    BC_REQUIRE(family >= 1 && family <= 3 && ws != nullptr, BC_ERR_ARG);
    return ccsdt_fused(family, d, t3, a, b, stream, eps_h, eps_p, ws);
}

int bc_ccsdt_s1_fused(const bc_tile_dims* d, double* t3, const double* const t1[9], const double* const v2[9],
                      void* stream) {
    return ccsdt_fused(3, d, t3, t1, v2, stream);
}
int bc_ccsdt_d1_tile(int variant, int tile, double* t3, const double* t2, const double* v2, void* stream) {
    const bc_tile_dims d{tile, tile, tile, tile, tile, tile, tile};
    return ccsdt_one(1, variant, &d, t3, t2, v2, stream);
}
int bc_ccsdt_d2_tile(int variant, int tile, double* t3, const double* t2, const double* v2, void* stream) {
    const bc_tile_dims d{tile, tile, tile, tile, tile, tile, tile};
    return ccsdt_one(2, variant, &d, t3, t2, v2, stream);
}

int bc_ccsdt_triples_energy(const bc_tile_dims* d, const double* const t1[9], const double* const v2s1[9],
                            const double* const t2d1[9], const double* const v2d1[9], const double* const t2d2[9],
                            const double* const v2d2[9], const double* eps_h, const double* eps_p, double* ws,
                            void* stream) {
    int st = check_dims(d, true);
    if (st) return st;
    BC_REQUIRE(t1 && v2s1 && t2d1 && v2d1 && t2d2 && v2d2 && eps_h && eps_p && ws, BC_ERR_ARG);
    BC_REQUIRE(d->h1 == d->h2 && d->h2 == d->h3 && d->p4 == d->p5 && d->p5 == d->p6, BC_ERR_UNSUPPORTED);
    BC_REQUIRE(d->k % 2 == 0 && d->h1 % 2 == 0 && d->h1 >= 12, BC_ERR_UNSUPPORTED);
    BC_REQUIRE(aligned(ws, 8) && aligned(eps_h, 8) && aligned(eps_p, 8), BC_ERR_ALIGN);
    const double* const* lists[6] = {t1, v2s1, t2d1, v2d1, t2d2, v2d2};
    for (int l = 0; l < 6; l += 2)
        for (int v = 0; v < 9; ++v) {
            if (!lists[l][v]) continue;
            BC_REQUIRE(lists[l + 1][v] != nullptr, BC_ERR_ARG);
            BC_REQUIRE(aligned(lists[l][v], 16) && aligned(lists[l + 1][v], 16), BC_ERR_ALIGN);
        }
    int e[7];
    dims_to_ext(d, e, true);
    return run_ccsdt_triples_energy(e, t1, v2s1, t2d1, v2d1, t2d2, v2d2, eps_h, eps_p, ws, as_stream(stream));
}

int bc_check_sumsq(int64_t n, const double* x, double* ws, void* stream) {
    BC_REQUIRE(n >= 0 && ws, BC_ERR_ARG);
    BC_REQUIRE(n == 0 || x, BC_ERR_ARG);
    BC_REQUIRE(aligned(ws, 8) && (n == 0 || aligned(x, 8)), BC_ERR_ALIGN);
    BC_REQUIRE(!overlap(ws, BC_CHECK_WS_DOUBLES * 8, x, (size_t)n * 8), BC_ERR_ALIAS);
    return run_sumsq(n, x, ws, as_stream(stream));
}

int bc_check_energy(const bc_tile_dims* d, const double* t3, const double* eps_h, const double* eps_p, double* ws,
                    void* stream) {
    int st = check_dims(d, false);
    if (st) return st;
    BC_REQUIRE(t3 && eps_h && eps_p && ws, BC_ERR_ARG);
    BC_REQUIRE(aligned(t3, 8) && aligned(eps_h, 8) && aligned(eps_p, 8) && aligned(ws, 8), BC_ERR_ALIGN);
    int e[7];
    dims_to_ext(d, e, false);
    BC_REQUIRE(!overlap(ws, BC_CHECK_WS_DOUBLES * 8, t3, t3_elems(e) * 8), BC_ERR_ALIAS);
    return run_energy(e, t3, eps_h, eps_p, ws, as_stream(stream));
}

int bc_fill(int kind, uint64_t seed, uint64_t tensor_id, uint64_t offset, int64_t n, double lo, double hi,
            double* out, void* stream) {
    BC_REQUIRE(kind >= 0 && kind <= 2 && n >= 0, BC_ERR_ARG);
    if (n == 0) return BC_OK;
    BC_REQUIRE(out != nullptr, BC_ERR_ARG);
    BC_REQUIRE(aligned(out, 8), BC_ERR_ALIGN);
    return run_fill<double>(kind, seed, tensor_id, offset, n, lo, hi, out, as_stream(stream));
}
int bc_fill_f32(int kind, uint64_t seed, uint64_t tensor_id, uint64_t offset, int64_t n, double lo, double hi,
                float* out, void* stream) {
    BC_REQUIRE(kind >= 0 && kind <= 2 && n >= 0, BC_ERR_ARG);
    if (n == 0) return BC_OK;
    BC_REQUIRE(out != nullptr, BC_ERR_ARG);
    BC_REQUIRE(aligned(out, 4), BC_ERR_ALIGN);
    return run_fill<float>(kind, seed, tensor_id, offset, n, lo, hi, out, as_stream(stream));
}

int bc_probe_fp64(int kind, int iters, double* scratch, int64_t scratch_doubles, double* flops, void* stream) {
    BC_REQUIRE((kind == 0 || kind == 1) && iters >= 1 && iters <= (1 << 20) && scratch && flops, BC_ERR_ARG);
    BC_REQUIRE(scratch_doubles >= probe_scratch_doubles(), BC_ERR_ARG);
    BC_REQUIRE(aligned(scratch, 8), BC_ERR_ALIGN);
    return run_probe_fp64(kind, iters, scratch, flops, as_stream(stream));
}
int64_t bc_probe_scratch_doubles(void) { return probe_scratch_doubles(); }

const char* bc_status_string(int status) {
    switch (status) {
        case BC_OK: return "BC_OK";
        case BC_ERR_ARG: return "BC_ERR_ARG: invalid argument";
        case BC_ERR_ALIGN: return "BC_ERR_ALIGN: pointer not sufficiently aligned";
        case BC_ERR_ALIAS: return "BC_ERR_ALIAS: output overlaps an input";
        case BC_ERR_UNSUPPORTED: return "BC_ERR_UNSUPPORTED: size beyond the compiled maximum";
        case BC_ERR_CUDA: return "BC_ERR_CUDA: CUDA launch failed (see bc_last_cuda_error)";
        default: return "unknown status";
    }
}
int bc_last_cuda_error(void) { return g_last_cuda_error; }
int bc_version(void) { return (0 << 16) | 1; }
int64_t bc_launch_count(void) { return g_launches; }
void bc_reset_launch_count(void) { g_launches = 0; }

}  // extern "C"
