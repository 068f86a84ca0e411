// ptx.cuh -- inline-PTX memory operations for the flag protocol (sm_100a).
//
// Memory-model reading (G6): the paper shows only a writer-side
// threadfence() before "get_value[i] <- true" (Alg.5 l.15-16)
// and is silent on the reader.  In the PTX model the pair we use is
//   producer:  st x[i] (weak)  ;  st.release.gpu flag[i] = epoch
//   consumer:  ld.acquire.gpu flag[j] == epoch  ;  ld.relaxed.gpu x[j]
// which synchronises-with and so guarantees the consumer's x load observes the
// producer's x store.  On sm_100a:
//   st.release.gpu  -> MEMBAR.ALL.GPU + STG.E.STRONG.GPU  (lighter than the
//                      paper's __threadfence(), which is MEMBAR.SC.GPU + CCTL)
//   ld.acquire.gpu  -> LDG.E.STRONG.GPU + CCTL.IVALL (L1 invalidate; the CSR
//                      slice lives in shared memory / registers, so the
//                      invalidate costs the solve nothing)
//   ld.relaxed.gpu  -> LDG.E.STRONG.GPU (served by L2, never a stale L1 line)
#pragma once
#include <cstdint>

namespace sptrsv_dev {

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ double ld_relaxed_f64(const double *p) {
    double v;
    asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// 16-byte vector accesses: each 8-byte element is single-copy atomic (the
// PROTO_FUSED record relies on exactly that, never on 16-byte atomicity).
__device__ __forceinline__ void ld_relaxed_v2_u64(const unsigned long long *p, unsigned long long &a,
                                                  unsigned long long &b) {
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

__device__ __forceinline__ void st_relaxed_v2_u64(unsigned long long *p, unsigned long long a,
                                                  unsigned long long b) {
    asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}

// Predicated forms: one store instruction guarded by a predicate register, so a
// single-lane store inside warp-uniform code does not open a divergent branch.
__device__ __forceinline__ void st_relaxed_v2_u64_if(bool pr, unsigned long long *p, unsigned long long a,
                                                     unsigned long long b) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};\n\t}" ::"l"(p),
                 "l"(a), "l"(b), "r"((unsigned)pr)
                 : "memory");
}
__device__ __forceinline__ void st_u64_if(bool pr, unsigned long long *p, unsigned long long v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q st.global.u64 [%0], %1;\n\t}" ::"l"(p), "l"(v),
                 "r"((unsigned)pr)
                 : "memory");
}

__device__ __forceinline__ void st_release_u32(uint32_t *p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ void st_relaxed_u32(uint32_t *p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ void st_relaxed_f64(double *p, double v) {
    asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}

__device__ __forceinline__ void st_relaxed_u64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void fence_acq_rel_gpu() {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

// L2 eviction policy for the once-read CSR stream (colidx, val, rowptr, b):
// evict_first keeps x and the flags -- re-read by every dependent -- in L2.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

// volatile: the compiler must not speculate these loads out of a guarding
// branch or ternary (a hoisted val[jd] with jd = -1 on an idle lane faults).
__device__ __forceinline__ int32_t ld_stream_i32(const int32_t *p, uint64_t pol) {
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;"
                 : "=r"(v) : "l"(p), "l"(pol));
    return v;
}

__device__ __forceinline__ double ld_stream_f64(const double *p, uint64_t pol) {
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;"
                 : "=d"(v) : "l"(p), "l"(pol));
    return v;
}

__device__ __forceinline__ void nanosleep_ns(uint32_t ns) {
    asm volatile("nanosleep.u32 %0;" ::"r"(ns));
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

}  // namespace sptrsv_dev
