// ptx.cuh -- memory-model primitives for the client<->server protocol.
//
// Cross-SM messages (request doorbells, responses, GTS, done flags) use the
// PTX memory model's release/acquire at .gpu scope: st.release.gpu lowers to
// MEMBAR.ALL.GPU + STG.STRONG.GPU, ld.acquire.gpu to LDG.STRONG.GPU +
// CCTL.IVALL (L1 invalidate), so payloads read after an acquire come from L2.
// Version-slot traffic uses .relaxed.gpu (morally strong, served by L2) so a
// reader racing a write-back sees either the old or the new 8-byte slot.
#pragma once
#include <cstdint>

namespace csmvd {

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint4 ld_relaxed_v4(const uint32_t* p) {
  uint4 v;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed64x2(uint64_t* p, uint64_t a, uint64_t b) {  // 16-byte aligned
  asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void fence_cta() {
  asm volatile("fence.acq_rel.cta;" ::: "memory");
}
__device__ __forceinline__ void fence_gpu() {
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// A version ring of NSLOT packed (ts << 32 | value) slots, one aligned
// record per item: NSLOT = 4 is a single 32-byte sector read by one 256-bit
// load (LDG.E.ENL2.256), NSLOT = 2 one 128-bit load.
template <int NSLOT>
struct Ring {
  uint64_t s[NSLOT];
};

template <int NSLOT>
__device__ __forceinline__ Ring<NSLOT> ld_ring(const uint64_t* p) {
  Ring<NSLOT> r;
#pragma unroll
  for (int j = 0; j < NSLOT; j += 4) {
    if (NSLOT - j >= 4) {
      asm volatile("ld.relaxed.gpu.global.v4.u64 {%0,%1,%2,%3}, [%4];"
                   : "=l"(r.s[j]), "=l"(r.s[j + 1]), "=l"(r.s[j + 2]), "=l"(r.s[j + 3])
                   : "l"(p + j)
                   : "memory");
    } else {
      asm volatile("ld.relaxed.gpu.global.v2.u64 {%0,%1}, [%2];"
                   : "=l"(r.s[j]), "=l"(r.s[j + 1])
                   : "l"(p + j)
                   : "memory");
    }
  }
  return r;
}

}  // namespace csmvd
