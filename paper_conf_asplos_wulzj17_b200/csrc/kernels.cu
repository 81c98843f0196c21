// kernels.cu — instantiates the wrapper and the unwrapped twins for every body and exposes a
// small dispatch table to the host runtime (runtime.cu). sm_100a only.
#include <cuda_runtime.h>
#include <type_traits>

#include "flep_device.cuh"
#include "bodies.cuh"
#include "gemm_tcgen05.cuh"
#include "stencil_tma.cuh"
#include "kernels.hpp"

#include <mutex>
#include <utility>

namespace flep {

namespace {

template <class Body>
struct Ops {
  static cudaError_t worker(const void* args, const WorkerParams& p, uint32_t W, cudaStream_t s,
                            bool cov) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    if (cov) flep_worker<Body, true><<<W, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    else flep_worker<Body, false><<<W, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    return cudaGetLastError();
  }
  static cudaError_t clc(const void* args, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    if constexpr (ClcRing<Body>::value) {
      if (clc_use_ring<Body>(p.poll)) {
        if (cov) flep_clc_ring<Body, true><<<N, Body::kThreads, Body::kDynSmem, s>>>(a, p);
        else flep_clc_ring<Body, false><<<N, Body::kThreads, Body::kDynSmem, s>>>(a, p);
        return cudaGetLastError();
      }
    }
    if (cov) flep_clc_worker<Body, true><<<N, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    else flep_clc_worker<Body, false><<<N, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    return cudaGetLastError();
  }
  static cudaError_t worker_sw(const void* args, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    if (cov) flep_worker_sw<Body, true><<<W, Body::kThreads + 32, Body::kDynSmem, s>>>(a, p);
    else flep_worker_sw<Body, false><<<W, Body::kThreads + 32, Body::kDynSmem, s>>>(a, p);
    return cudaGetLastError();
  }
  static cudaError_t occupancy_sw(int* k, bool cov) {
    if (cov) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker_sw<Body, true>, Body::kThreads + 32, Body::kDynSmem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker_sw<Body, false>, Body::kThreads + 32, Body::kDynSmem);
  }
  static cudaError_t warp_worker(const void* args, const WorkerParams& p, uint32_t G, cudaStream_t s, bool cov) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    if (cov) flep_warp_worker<Body, true><<<G, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    else flep_warp_worker<Body, false><<<G, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    return cudaGetLastError();
  }
  static cudaError_t worker_ic(const void* args, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    if (cov) flep_worker_ic<Body, true><<<W, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    else flep_worker_ic<Body, false><<<W, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    return cudaGetLastError();
  }
  static cudaError_t occupancy_ic(int* k, bool cov) {
    if (cov) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker_ic<Body, true>, Body::kThreads, Body::kDynSmem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker_ic<Body, false>, Body::kThreads, Body::kDynSmem);
  }
  static cudaError_t occupancy_warp(int* k, bool cov) {
    if (cov) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_warp_worker<Body, true>, Body::kThreads, Body::kDynSmem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_warp_worker<Body, false>, Body::kThreads, Body::kDynSmem);
  }
  static cudaError_t unwrapped(const void* args, dim3 grid, uint32_t offset, uint32_t count,
                               cudaStream_t s) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    if (count == 0) flep_unwrapped<Body><<<grid, Body::kThreads, Body::kDynSmem, s>>>(a, grid.x, grid.y, 0);
    else flep_unwrapped<Body><<<count, Body::kThreads, Body::kDynSmem, s>>>(a, grid.x, grid.y, offset);
    return cudaGetLastError();
  }
  static cudaError_t sliced(const void* args, dim3 grid, uint32_t offset, uint32_t count, const SliceParams& sp,
                            cudaStream_t s) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    flep_slice<Body><<<count, Body::kThreads, Body::kDynSmem, s>>>(a, grid.x, grid.y, offset, sp);
    return cudaGetLastError();
  }
  static cudaError_t static_launch(const void* args, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s) {
    const typename Body::Args& a = *reinterpret_cast<const typename Body::Args*>(args);
    WorkerParams p{};
    p.static_sched = 1u;
    p.n_blocks = grid.x * grid.y * grid.z;
    p.chunk = chunk ? chunk : 1u;
    p.workers = ctas;
    p.gx = grid.x;
    p.gy = grid.y;
    flep_static<Body><<<ctas, Body::kThreads, Body::kDynSmem, s>>>(a, p);
    return cudaGetLastError();
  }
  static cudaError_t occupancy(int* k, bool cov) {
    cudaError_t e;
    if (Body::kDynSmem > 48 * 1024) {
      e = cudaFuncSetAttribute(flep_worker<Body, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
      if (e) return e;
      e = cudaFuncSetAttribute(flep_worker<Body, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
      if (e) return e;
      e = cudaFuncSetAttribute(flep_unwrapped<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
      if (e) return e;
    }
    if (cov) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker<Body, true>, Body::kThreads, Body::kDynSmem);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker<Body, false>, Body::kThreads, Body::kDynSmem);
  }
};

// Adapter: bodies written without kDynSmem get 0.
template <class B>
struct WithSmem : B {
  static constexpr size_t kDynSmem = 0;
};

}  // namespace

// GEMM launchers live in gemm_tcgen05.cu (they need the tensor-map encoder); they use these.
// dynamic shared memory of a launch whose chunks hold `chunk` blocks (bodies may size it by C)
template <class B, class = void> struct HasDynSmemFn : std::false_type {};
template <class B> struct HasDynSmemFn<B, std::void_t<decltype(B::dyn_smem(1u))>> : std::true_type {};
template <class Body>
constexpr size_t smem_for(uint32_t chunk) {
  if constexpr (HasDynSmemFn<Body>::value) return Body::dyn_smem(chunk);
  else return Body::kDynSmem;
}
template <class Body>
cudaError_t launch_worker_raw(const typename Body::Args& a, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov) {
  const size_t sm = smem_for<Body>(p.chunk);
  if (cov) flep_worker<Body, true><<<W, Body::kThreads, sm, s>>>(a, p);
  else flep_worker<Body, false><<<W, Body::kThreads, sm, s>>>(a, p);
  return cudaGetLastError();
}
template <class Body>
cudaError_t launch_unwrapped_raw(const typename Body::Args& a, dim3 grid, uint32_t offset, uint32_t count, cudaStream_t s) {
  const size_t sm = smem_for<Body>(1);
  if (count == 0) flep_unwrapped<Body><<<grid, Body::kThreads, sm, s>>>(a, grid.x, grid.y, 0);
  else flep_unwrapped<Body><<<count, Body::kThreads, sm, s>>>(a, grid.x, grid.y, offset);
  return cudaGetLastError();
}
template <class Body>
cudaError_t occupancy_raw(int* k, bool cov) {
  cudaError_t e;
  if (Body::kDynSmem > 48 * 1024) {
    e = cudaFuncSetAttribute(flep_worker<Body, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
    if (e) return e;
    e = cudaFuncSetAttribute(flep_worker<Body, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
    if (e) return e;
    e = cudaFuncSetAttribute(flep_unwrapped<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
    if (e) return e;
    if constexpr (!Body::kPersistent) {
      e = cudaFuncSetAttribute(flep_clc_worker<Body, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
      if (e) return e;
      e = cudaFuncSetAttribute(flep_clc_worker<Body, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Body::kDynSmem);
      if (e) return e;
    }
  }
  if (cov) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker<Body, true>, Body::kThreads, Body::kDynSmem);
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker<Body, false>, Body::kThreads, Body::kDynSmem);
}
template <class Body>
cudaError_t launch_slice_raw(const typename Body::Args& a, dim3 grid, uint32_t offset, uint32_t count,
                             const SliceParams& sp, cudaStream_t s) {
  const size_t sm = smem_for<Body>(1);
  if (sm > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(flep_slice<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e) return e;
  }
  flep_slice<Body><<<count, Body::kThreads, sm, s>>>(a, grid.x, grid.y, offset, sp);
  return cudaGetLastError();
}
template <class Body>
cudaError_t launch_static_raw(const typename Body::Args& a, dim3 grid, uint32_t ctas, uint32_t chunk, cudaStream_t s) {
  const size_t sm = smem_for<Body>(chunk ? chunk : 1u);
  if (sm > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(flep_static<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e) return e;
  }
  WorkerParams p{};
  p.static_sched = 1u;
  p.n_blocks = grid.x * grid.y * grid.z;
  p.chunk = chunk ? chunk : 1u;
  p.workers = ctas;
  p.gx = grid.x;
  p.gy = grid.y;
  flep_static<Body><<<ctas, Body::kThreads, sm, s>>>(a, p);
  return cudaGetLastError();
}
template <class Body>
cudaError_t launch_clc_raw(const typename Body::Args& a, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov) {
  const size_t sm = smem_for<Body>(p.chunk);
  if (cov) flep_clc_worker<Body, true><<<N, Body::kThreads, sm, s>>>(a, p);
  else flep_clc_worker<Body, false><<<N, Body::kThreads, sm, s>>>(a, p);
  return cudaGetLastError();
}
template cudaError_t launch_worker_raw<Stencil5TmaBody>(const Stencil5TmaBody::Args&, const WorkerParams&, uint32_t, cudaStream_t, bool);
template cudaError_t launch_unwrapped_raw<Stencil5TmaBody>(const Stencil5TmaBody::Args&, dim3, uint32_t, uint32_t, cudaStream_t);
template cudaError_t launch_clc_raw<Stencil5TmaBody>(const Stencil5TmaBody::Args&, const WorkerParams&, uint32_t, cudaStream_t, bool);
template cudaError_t occupancy_raw<Stencil5TmaBody>(int*, bool);
template cudaError_t launch_worker_raw<GemmBody>(const GemmBody::Args&, const WorkerParams&, uint32_t, cudaStream_t, bool);
template cudaError_t launch_unwrapped_raw<GemmBody>(const GemmBody::Args&, dim3, uint32_t, uint32_t, cudaStream_t);
template cudaError_t occupancy_raw<GemmBody>(int*, bool);
template cudaError_t launch_static_raw<GemmBody>(const GemmBody::Args&, dim3, uint32_t, uint32_t, cudaStream_t);
template cudaError_t launch_slice_raw<GemmBody>(const GemmBody::Args&, dim3, uint32_t, uint32_t, const SliceParams&, cudaStream_t);
template cudaError_t launch_slice_raw<Stencil5TmaBody>(const Stencil5TmaBody::Args&, dim3, uint32_t, uint32_t, const SliceParams&, cudaStream_t);

namespace {

using SaxpyI32 = WithSmem<SaxpyBody<true>>;
using SaxpyF32 = WithSmem<SaxpyBody<false>>;
using Spmv = WithSmem<SpmvBody>;
using SpmvVec = WithSmem<SpmvVecBody>;
using StencilF32 = WithSmem<Stencil5Body<false>>;
using StencilI32 = WithSmem<Stencil5Body<true>>;

const BodyOps kOps[] = {
    {0, 0, 0, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr},
    {FLEP_BODY_SAXPY_I32, SaxpyI32::kThreads, sizeof(flep_saxpy_i32_args), &Ops<SaxpyI32>::worker,
     &Ops<SaxpyI32>::unwrapped, &Ops<SaxpyI32>::occupancy, nullptr, &Ops<SaxpyI32>::clc,
     &Ops<SaxpyI32>::worker_sw, &Ops<SaxpyI32>::occupancy_sw, nullptr, nullptr, 0, &Ops<SaxpyI32>::sliced, &Ops<SaxpyI32>::static_launch, nullptr, &Ops<SaxpyI32>::worker_ic, &Ops<SaxpyI32>::occupancy_ic},
    {FLEP_BODY_SAXPY_F32, SaxpyF32::kThreads, sizeof(flep_saxpy_f32_args), &Ops<SaxpyF32>::worker,
     &Ops<SaxpyF32>::unwrapped, &Ops<SaxpyF32>::occupancy, nullptr, &Ops<SaxpyF32>::clc,
     &Ops<SaxpyF32>::worker_sw, &Ops<SaxpyF32>::occupancy_sw, nullptr, nullptr, 0, &Ops<SaxpyF32>::sliced, &Ops<SaxpyF32>::static_launch, nullptr, &Ops<SaxpyF32>::worker_ic, &Ops<SaxpyF32>::occupancy_ic},
    {FLEP_BODY_SPMV_CSR_F32, Spmv::kThreads, sizeof(flep_spmv_args), &Ops<Spmv>::worker,
     &Ops<Spmv>::unwrapped, &Ops<Spmv>::occupancy, nullptr, &Ops<Spmv>::clc,
     &Ops<Spmv>::worker_sw, &Ops<Spmv>::occupancy_sw, nullptr, nullptr, 0, &Ops<Spmv>::sliced, &Ops<Spmv>::static_launch, nullptr, &Ops<Spmv>::worker_ic, &Ops<Spmv>::occupancy_ic},
    {FLEP_BODY_STENCIL5_F32, StencilF32::kThreads, sizeof(flep_stencil_args), &Ops<StencilF32>::worker,
     &Ops<StencilF32>::unwrapped, &Ops<StencilF32>::occupancy, nullptr, &Ops<StencilF32>::clc,
     &Ops<StencilF32>::worker_sw, &Ops<StencilF32>::occupancy_sw, &Ops<StencilF32>::warp_worker,
     &Ops<StencilF32>::occupancy_warp, StencilF32::kWarpTasks, &Ops<StencilF32>::sliced, &Ops<StencilF32>::static_launch, nullptr, &Ops<StencilF32>::worker_ic, &Ops<StencilF32>::occupancy_ic},
    {FLEP_BODY_STENCIL5_I32, StencilI32::kThreads, sizeof(flep_stencil_args), &Ops<StencilI32>::worker,
     &Ops<StencilI32>::unwrapped, &Ops<StencilI32>::occupancy, nullptr, &Ops<StencilI32>::clc,
     &Ops<StencilI32>::worker_sw, &Ops<StencilI32>::occupancy_sw, &Ops<StencilI32>::warp_worker,
     &Ops<StencilI32>::occupancy_warp, StencilI32::kWarpTasks, &Ops<StencilI32>::sliced, &Ops<StencilI32>::static_launch, nullptr, &Ops<StencilI32>::worker_ic, &Ops<StencilI32>::occupancy_ic},
    {FLEP_BODY_GEMM_BF16, GemmBody::kThreads, sizeof(flep_gemm_args), &gemm_worker_launch,
     &gemm_unwrapped_launch, &gemm_occupancy, &gemm_validate, nullptr, nullptr, nullptr, nullptr, nullptr, 0,
     &gemm_slice_launch, &gemm_static_launch, nullptr},
    {FLEP_BODY_STENCIL5_F32_TMA, Stencil5TmaBody::kThreads, sizeof(flep_stencil_args), &stencil_tma_worker_launch,
     &stencil_tma_unwrapped_launch, &stencil_tma_occupancy, &stencil_tma_validate, &stencil_tma_clc_launch,
     nullptr, nullptr, nullptr, nullptr, 0, &stencil_tma_slice_launch},
    {FLEP_BODY_SPMV_CSR_F32_VEC, SpmvVec::kThreads, sizeof(flep_spmv_args), &Ops<SpmvVec>::worker,
     &Ops<SpmvVec>::unwrapped, &Ops<SpmvVec>::occupancy, nullptr, &Ops<SpmvVec>::clc,
     &Ops<SpmvVec>::worker_sw, &Ops<SpmvVec>::occupancy_sw, &Ops<SpmvVec>::warp_worker,
     &Ops<SpmvVec>::occupancy_warp, SpmvVec::kWarpTasks, &Ops<SpmvVec>::sliced, &Ops<SpmvVec>::static_launch, nullptr, &Ops<SpmvVec>::worker_ic, &Ops<SpmvVec>::occupancy_ic},
    {FLEP_BODY_GEMM_BF16_2SM, 256 /* Gemm2::kThreads (gemm2_tcgen05.cuh, its own TU) */, sizeof(flep_gemm_args), &gemm2_worker_launch,
     &gemm2_unwrapped_launch, &gemm2_occupancy, &gemm2_validate, nullptr, nullptr, nullptr, nullptr, nullptr, 0,
     &gemm2_slice_launch, &gemm2_static_launch, &gemm2_max_pairs},
    {FLEP_BODY_GEMM_BF16_2SM_W, 256 /* Gemm2W::kThreads */, sizeof(flep_gemm_args), &gemm2w_worker_launch,
     &gemm2w_unwrapped_launch, &gemm2w_occupancy, &gemm2w_validate, nullptr, nullptr, nullptr, nullptr, nullptr, 0,
     &gemm2w_slice_launch, &gemm2w_static_launch, &gemm2w_max_pairs, nullptr, nullptr, 2},
};

}  // namespace

#ifdef FLEP_TRACE
cudaError_t set_unwrapped_trace(uint64_t* p) {
  return cudaMemcpyToSymbol(g_unwrapped_trace, &p, sizeof(p));
}
#endif

// ---- user-defined bodies (flep_register_body): a fixed table of FLEP_BODY_USER_MAX slots whose
// BodyOps entries are thunks into the caller's C launchers (plain function pointers, no captures)
namespace {
flep_body_ops g_user_tab[FLEP_BODY_USER_MAX];
BodyOps g_user_ops[FLEP_BODY_USER_MAX];
int g_user_n = 0;
std::mutex g_user_mu;

template <int I>
cudaError_t u_worker(const void* a, const WorkerParams& p, uint32_t W, cudaStream_t s, bool cov) {
  return static_cast<cudaError_t>(g_user_tab[I].worker(a, &p, W, static_cast<flep_stream_t>(s), cov ? 1 : 0));
}
template <int I>
cudaError_t u_unwrapped(const void* a, dim3 g, uint32_t offset, uint32_t count, cudaStream_t s) {
  const flep_dim3 d = {g.x, g.y, g.z};
  return static_cast<cudaError_t>(g_user_tab[I].unwrapped(a, d, offset, count, static_cast<flep_stream_t>(s)));
}
template <int I>
cudaError_t u_static(const void* a, dim3 g, uint32_t ctas, uint32_t chunk, cudaStream_t s) {
  const flep_dim3 d = {g.x, g.y, g.z};
  return static_cast<cudaError_t>(g_user_tab[I].static_launch(a, d, ctas, chunk, static_cast<flep_stream_t>(s)));
}
template <int I>
cudaError_t u_clc(const void* a, const WorkerParams& p, uint32_t N, cudaStream_t s, bool cov) {
  return static_cast<cudaError_t>(g_user_tab[I].clc(a, &p, N, static_cast<flep_stream_t>(s), cov ? 1 : 0));
}
template <int I>
cudaError_t u_sliced(const void* a, dim3 g, uint32_t offset, uint32_t count, const SliceParams& sp, cudaStream_t s) {
  const flep_dim3 d = {g.x, g.y, g.z};
  return static_cast<cudaError_t>(g_user_tab[I].sliced(a, d, offset, count, &sp, static_cast<flep_stream_t>(s)));
}
template <int I>
cudaError_t u_occupancy(int* k, bool cov) {
  return static_cast<cudaError_t>(g_user_tab[I].occupancy(k, cov ? 1 : 0));
}
template <int I>
void make_user_ops(BodyOps& o) {
  o = BodyOps{};
  o.body = FLEP_BODY_USER_FIRST + I;
  o.threads = static_cast<int>(g_user_tab[I].threads);
  o.args_size = g_user_tab[I].args_size;
  o.worker = &u_worker<I>;
  o.unwrapped = &u_unwrapped<I>;
  o.occupancy = &u_occupancy<I>;
  o.static_launch = g_user_tab[I].static_launch ? &u_static<I> : nullptr;
  o.clc = g_user_tab[I].clc ? &u_clc<I> : nullptr;
  o.sliced = g_user_tab[I].sliced ? &u_sliced<I> : nullptr;
}
template <int... I>
void make_user_ops_at(int slot, std::integer_sequence<int, I...>) {
  ((slot == I ? make_user_ops<I>(g_user_ops[I]) : void()), ...);
}
}  // namespace

int32_t register_user_body(const flep_body_ops* o, const char** why) {
  if (!o || !o->worker || !o->unwrapped || !o->occupancy) { *why = "incomplete flep_body_ops"; return -1; }
  if (o->abi_version != FLEP_BODY_ABI_VERSION) { *why = "abi_version mismatch"; return -1; }
  if (o->threads == 0 || o->threads > 1024 || o->args_size == 0) { *why = "threads / args_size out of range"; return -1; }
  std::lock_guard<std::mutex> lk(g_user_mu);
  if (g_user_n >= FLEP_BODY_USER_MAX) { *why = "all FLEP_BODY_USER_MAX user body slots are taken"; return -2; }
  const int slot = g_user_n;
  g_user_tab[slot] = *o;
  make_user_ops_at(slot, std::make_integer_sequence<int, FLEP_BODY_USER_MAX>{});
  g_user_n = slot + 1;                     // published after the entry is complete
  return FLEP_BODY_USER_FIRST + slot;
}

const BodyOps* body_ops(int32_t body) {
  if (body >= FLEP_BODY_USER_FIRST && body < FLEP_BODY_USER_FIRST + FLEP_BODY_USER_MAX) {
    std::lock_guard<std::mutex> lk(g_user_mu);
    return body - FLEP_BODY_USER_FIRST < g_user_n ? &g_user_ops[body - FLEP_BODY_USER_FIRST] : nullptr;
  }
  if (body < 1 || body > FLEP_BODY_GEMM_BF16_2SM_W) return nullptr;
  return &kOps[body];
}

}  // namespace flep
