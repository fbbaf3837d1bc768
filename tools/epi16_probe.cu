// Microbenchmark: the engine's identity-F epilogue (TMEM -> +bias -> bf16 ->
// smem transpose -> coalesced global stores) of one 128 x 256 fp32
// accumulator per CTA, with NW epilogue warps (NW / 4 per TMEM lane quarter)
// draining W-column chunks, while another warp keeps the tensor core busy on
// the other TMEM half (as in the engine's double-buffered mainloop).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_eurosys_ohlks22_b200/csrc \
//        -o tools/epi16_probe tools/epi16_probe.cu
#include <cstdio>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "tc_common.cuh"

using namespace ooo::tc;

__device__ __forceinline__ void tmem_ld16_issue(uint32_t a, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(a));
}
__device__ __forceinline__ void tmem_ld16_wait(uint32_t (&r)[16]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]), "+r"(r[7]),
                 "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]), "+r"(r[14]),
                 "+r"(r[15])
               :
               : "memory");
}
// 32 rows x 16 bf16 columns (lane = row) through a 1 KiB per-warp buffer:
// 16-B chunk c of 32-B row r at chunk c ^ ((r >> 2) & 1) (conflict-free),
// read back as 2 lanes per row -> 32-B row segments.
__device__ __forceinline__ void store16_rows_packed(__nv_bfloat16 *g, int ldc, uint32_t buf, int lane,
                                                    const uint32_t (&u)[8], int col0, int row0) {
  __syncwarp();
  const uint32_t rb = buf + lane * 32;
#pragma unroll
  for (int c = 0; c < 2; ++c) {
    const uint32_t a = rb + ((c ^ ((lane >> 2) & 1)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(u[4 * c]), "r"(u[4 * c + 1]),
                 "r"(u[4 * c + 2]), "r"(u[4 * c + 3])
                 : "memory");
  }
  __syncwarp();
  const int c = lane & 1;
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const int r = (lane >> 1) + 16 * k;
    uint32_t x, y, z, w;
    asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(x), "=r"(y), "=r"(z), "=r"(w)
                 : "r"(buf + r * 32 + ((c ^ ((r >> 2) & 1)) << 4))
                 : "memory");
    *reinterpret_cast<uint4 *>(g + (size_t)(row0 + r) * ldc + col0 + c * 8) = make_uint4(x, y, z, w);
  }
}

template <int NW, int W>
__global__ void __launch_bounds__(NW * 32 + 32, 1) epi(__nv_bfloat16 *out, int ldc, int tiles, long long *cyc) {
  __shared__ __align__(1024) uint8_t stg_all[NW * 32 * W * 2];
  __shared__ float bias_s[256];
  __shared__ uint32_t tslot;
  __shared__ __align__(1024) uint8_t opnd[16384];
  __shared__ __align__(8) uint64_t mbar;
  __shared__ volatile int stop;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { stop = 0; mbar_init(smem_u32(&mbar), 1); }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tslot)), "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (threadIdx.x < 256) bias_s[threadIdx.x] = 0.25f * threadIdx.x;
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = tslot;
  if (warp == NW) {
    if (lane == 0) {
      const uint32_t ID = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(128 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
      const uint64_t ad = sdesc(smem_u32(opnd), 16, 1024);
      uint32_t ph = 0;
      while (!stop) {
        for (int k = 0; k < 4; ++k) umma_bf16(tmem + 256, ad + 2 * k, ad + 2 * k, ID, k ? 1u : 0u);
        umma_commit(smem_u32(&mbar));
        mbar_wait(smem_u32(&mbar), ph);
        ph ^= 1;
      }
    }
    __syncwarp();
  } else {
    constexpr int PER = NW / 4, NCH = 256 / W;
    const int q = warp & 3, h = warp >> 2;
    const uint32_t stg = smem_u32(stg_all) + warp * 32 * W * 2;
    const int row0 = blockIdx.x * 128 + q * 32;
    const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16);
    long long t0 = clock64();
    for (int tile = 0; tile < tiles; ++tile) {
      uint32_t ra[W];
      if (W == 32) tmem_ld32_issue(tbase + (uint32_t)(h * 32), *reinterpret_cast<uint32_t(*)[32]>(ra));
      else tmem_ld16_issue(tbase + (uint32_t)(h * 16), *reinterpret_cast<uint32_t(*)[16]>(ra));
      for (int c = h; c < NCH; c += PER) {
        const int col0 = (tile % 3) * 256 + c * W;
        if (W == 32) tmem_ld_wait(*reinterpret_cast<uint32_t(*)[32]>(ra));
        else tmem_ld16_wait(*reinterpret_cast<uint32_t(*)[16]>(ra));
        float v[W];
#pragma unroll
        for (int i = 0; i < W; ++i) v[i] = __uint_as_float(ra[i]);
        if (c + PER < NCH) {
          if (W == 32) tmem_ld32_issue(tbase + (uint32_t)((c + PER) * 32), *reinterpret_cast<uint32_t(*)[32]>(ra));
          else tmem_ld16_issue(tbase + (uint32_t)((c + PER) * 16), *reinterpret_cast<uint32_t(*)[16]>(ra));
        }
#pragma unroll
        for (int i = 0; i < W; ++i) v[i] += bias_s[c * W + i];
        uint32_t u[W / 2];
#pragma unroll
        for (int j = 0; j < W / 2; ++j) u[j] = pack_bf2(v[2 * j], v[2 * j + 1]);
        if (W == 32) store32_rows_packed(out, ldc, stg, lane, *reinterpret_cast<uint32_t(*)[16]>(u), col0, row0, 1 << 30);
        else store16_rows_packed(out, ldc, stg, lane, *reinterpret_cast<uint32_t(*)[8]>(u), col0, row0);
      }
      asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
    }
    if (threadIdx.x == 0) { cyc[blockIdx.x] = clock64() - t0; stop = 1; }
  }
  fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
}

template <int NW, int W>
void run(__nv_bfloat16 *out, int ldc, long long *d) {
  const int tiles = 200;
  epi<NW, W><<<148, NW * 32 + 32>>>(out, ldc, tiles, d);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  double m = 0;
  for (int i = 0; i < 148; ++i) m += h[i];
  m /= 148;
  printf("%2d epilogue warps, %2d-column chunks: %6.0f cycles per 128x256 tile (MMA running)  (%s)\n", NW, W, m / tiles,
         cudaGetErrorString(e));
}

int main() {
  __nv_bfloat16 *out;
  const int ldc = 768, rows = 148 * 128;
  cudaMalloc(&out, (size_t)rows * ldc * 2);
  long long *d;
  cudaMalloc(&d, 148 * 8);
  run<8, 32>(out, ldc, d);
  run<8, 16>(out, ldc, d);

  run<16, 16>(out, ldc, d);
  return 0;
}
