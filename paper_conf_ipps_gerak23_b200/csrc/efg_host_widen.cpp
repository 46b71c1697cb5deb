// efg_host_widen.cpp — host side of the compact depth transfer (efg_bfs with a
// host depth array): one byte per vertex crosses PCIe and the host widens it
// to the caller's int32 array.  The widening is bound by host memory writes;
// streaming (non-temporal) stores skip the read-for-ownership of the
// destination lines, which a plain store loop pays on every line.
#include <immintrin.h>
#include <omp.h>

#include <cstdint>

#include "efg_internal.h"

namespace efg {
namespace {

__attribute__((target("avx2"))) void widen_avx2(const int8_t *s, int32_t *d, int64_t n)
{
    int64_t i = 0;
    for (; i < n && (reinterpret_cast<uintptr_t>(d + i) & 31); ++i) d[i] = s[i];
    for (; i + 8 <= n; i += 8) {
        const __m128i b = _mm_loadl_epi64(reinterpret_cast<const __m128i *>(s + i));
        _mm256_stream_si256(reinterpret_cast<__m256i *>(d + i), _mm256_cvtepi8_epi32(b));
    }
    for (; i < n; ++i) d[i] = s[i];
    _mm_sfence();
}

void widen_plain(const int8_t *s, int32_t *d, int64_t n)
{
    for (int64_t i = 0; i < n; ++i) d[i] = s[i];
}

// 4-bit codes: vertex i of the range is nibble i & 7 of word i >> 3, depth = code - 1
__attribute__((target("avx2"))) void widen4_avx2(const uint32_t *w, int32_t *d, int64_t n)
{
    const __m256i sh = _mm256_setr_epi32(0, 4, 8, 12, 16, 20, 24, 28);
    const __m256i m15 = _mm256_set1_epi32(15), one = _mm256_set1_epi32(1);
    const bool aligned = (reinterpret_cast<uintptr_t>(d) & 31) == 0;
    int64_t g = 0;
    for (; 8 * g + 8 <= n; ++g) {
        __m256i v = _mm256_srlv_epi32(_mm256_set1_epi32((int)w[g]), sh);
        v = _mm256_sub_epi32(_mm256_and_si256(v, m15), one);
        if (aligned)
            _mm256_stream_si256(reinterpret_cast<__m256i *>(d + 8 * g), v);
        else
            _mm256_storeu_si256(reinterpret_cast<__m256i *>(d + 8 * g), v);
    }
    for (int64_t i = 8 * g; i < n; ++i) d[i] = (int32_t)((w[i >> 3] >> (4 * (i & 7))) & 15u) - 1;
    _mm_sfence();
}

void widen4_plain(const uint32_t *w, int32_t *d, int64_t n)
{
    for (int64_t i = 0; i < n; ++i) d[i] = (int32_t)((w[i >> 3] >> (4 * (i & 7))) & 15u) - 1;
}

}  // namespace

void host_widen_i8_i32(const int8_t *src, int32_t *dst, int64_t n)
{
    static const bool avx2 = __builtin_cpu_supports("avx2");
#pragma omp parallel
    {
        const int t = omp_get_thread_num(), nt = omp_get_num_threads();
        const int64_t a = (n * t / nt) & ~int64_t(63), b = t == nt - 1 ? n : (n * (t + 1) / nt) & ~int64_t(63);
        if (b > a) {
            if (avx2)
                widen_avx2(src + a, dst + a, b - a);
            else
                widen_plain(src + a, dst + a, b - a);
        }
    }
}

void host_widen_u4_i32(const uint32_t *src, int32_t *dst, int64_t n)
{
    static const bool avx2 = __builtin_cpu_supports("avx2");
#pragma omp parallel
    {
        const int t = omp_get_thread_num(), nt = omp_get_num_threads();
        const int64_t a = (n * t / nt) & ~int64_t(63), b = t == nt - 1 ? n : (n * (t + 1) / nt) & ~int64_t(63);
        if (b > a) {
            if (avx2)
                widen4_avx2(src + a / 8, dst + a, b - a);
            else
                widen4_plain(src + a / 8, dst + a, b - a);
        }
    }
}

}  // namespace efg
