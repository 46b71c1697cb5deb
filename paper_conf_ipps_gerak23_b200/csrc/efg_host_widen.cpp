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

}  // namespace efg
