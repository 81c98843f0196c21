// flep_body.cuh — writing your own preemptable kernel body (the user-defined body extension of
// include/flep.h, flep_register_body). The paper's compiler turns any kernel into its
// persistent-thread form (Fig. 4); here a kernel is written once as a body and this header
// instantiates, in the caller's own .cu (compiled for sm_100a against the same headers as
// libflep.so), the three grids the runtime needs:
//   * the FLEP worker (flep_worker<Body>): resident CTAs pull chunks of original block indices
//     from the launch's counter, poll the control word every K chunks and yield (temporal or
//     spatial), exactly-once across preempt/resume;
//   * the original kernel (flep_unwrapped<Body>): one CTA per original block;
//   * the static persistent twin (flep_static<Body>): the overhead baseline;
//   * the CLC worker (flep_clc_worker<Body>, FLEP_KFLAG_CLC) and the device-checked slice kernel
//     (flep_slice<Body>, FLEP_POLICY_SLICE_DEVICE).
//
// A body is a struct with
//   using Args = <trivially copyable argument struct, passed by value to the grids>;
//   static constexpr int kThreads;      // CTA size
//   static constexpr int kMinBlocks;    // __launch_bounds__ min blocks per SM: give the original
//                                       // grid's occupancy, so that the worker (which holds more
//                                       // state) is register-capped to the same CTAs per SM
//   __device__ static void run(const Args&, uint32_t b0, uint32_t b1, uint32_t gx, uint32_t gy);
//                                       // run original blocks [b0, b1) of a gx x gy grid; every
//                                       // thread of the CTA calls it; a block's result must not
//                                       // depend on which CTA or SM runs it
// and setup/teardown/kPersistent, inherited from flep::UserBody for bodies without per-worker
// resources. A body whose run() uses no shared memory and no CTA barrier may declare
//   static constexpr uint32_t kWarpTasks = kThreads / 32;
// and then runs, with the CLC fetch at K <= 2, without a CTA barrier between blocks (flep_clc_ring). Then, at namespace scope:
//   FLEP_DEFINE_BODY(my_body, MyBody)
// defines extern "C" void my_body_ops(flep_body_ops* out), which fills the table that
// flep_register_body(rt, &ops, &body_id) takes; body_id is then used in flep_kernel_desc.body.
// Dynamic shared memory is not supported for user bodies (static __shared__ inside run is).
#pragma once
#include <cuda_runtime.h>

#include "flep.h"
#include "../paper_conf_asplos_wulzj17_b200/csrc/flep_device.cuh"

namespace flep {

using UserBody = NoResources;        // not persistent, no per-worker setup/teardown

template <class Body>
int user_worker_launch(const void* a, const void* wp, uint32_t W, flep_stream_t s, int cov) {
  const auto& args = *static_cast<const typename Body::Args*>(a);
  const auto& p = *static_cast<const WorkerParams*>(wp);
  const cudaStream_t st = static_cast<cudaStream_t>(s);
  if (cov) flep_worker<Body, true><<<W, Body::kThreads, 0, st>>>(args, p);
  else flep_worker<Body, false><<<W, Body::kThreads, 0, st>>>(args, p);
  return static_cast<int>(cudaGetLastError());
}

template <class Body>
int user_unwrapped_launch(const void* a, flep_dim3 g, uint32_t offset, uint32_t count, flep_stream_t s) {
  const auto& args = *static_cast<const typename Body::Args*>(a);
  const cudaStream_t st = static_cast<cudaStream_t>(s);
  if (count == 0) flep_unwrapped<Body><<<dim3(g.x, g.y, g.z), Body::kThreads, 0, st>>>(args, g.x, g.y, 0);
  else flep_unwrapped<Body><<<count, Body::kThreads, 0, st>>>(args, g.x, g.y, offset);
  return static_cast<int>(cudaGetLastError());
}

template <class Body>
int user_static_launch(const void* a, flep_dim3 g, uint32_t ctas, uint32_t chunk, flep_stream_t s) {
  const auto& args = *static_cast<const typename Body::Args*>(a);
  WorkerParams p{};
  p.static_sched = 1u;
  p.n_blocks = g.x * g.y * g.z;
  p.chunk = chunk ? chunk : 1u;
  p.workers = ctas;
  p.gx = g.x;
  p.gy = g.y;
  flep_static<Body><<<ctas, Body::kThreads, 0, static_cast<cudaStream_t>(s)>>>(args, p);
  return static_cast<int>(cudaGetLastError());
}

template <class Body>
int user_occupancy(int* k, int cov) {
  return static_cast<int>(cov ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker<Body, true>, Body::kThreads, 0)
                              : cudaOccupancyMaxActiveBlocksPerMultiprocessor(k, flep_worker<Body, false>, Body::kThreads, 0));
}

template <class Body>
int user_clc_launch(const void* a, const void* wp, uint32_t N, flep_stream_t s, int cov) {
  const auto& args = *static_cast<const typename Body::Args*>(a);
  const auto& p = *static_cast<const WorkerParams*>(wp);
  const cudaStream_t st = static_cast<cudaStream_t>(s);
  if constexpr (ClcRing<Body>::value) {
    if (clc_use_ring<Body>(p.poll)) {
      if (cov) flep_clc_ring<Body, true><<<N, Body::kThreads, 0, st>>>(args, p);
      else flep_clc_ring<Body, false><<<N, Body::kThreads, 0, st>>>(args, p);
      return static_cast<int>(cudaGetLastError());
    }
  }
  if (cov) flep_clc_worker<Body, true><<<N, Body::kThreads, 0, st>>>(args, p);
  else flep_clc_worker<Body, false><<<N, Body::kThreads, 0, st>>>(args, p);
  return static_cast<int>(cudaGetLastError());
}

template <class Body>
int user_slice_launch(const void* a, flep_dim3 g, uint32_t offset, uint32_t count, const void* sp, flep_stream_t s) {
  const auto& args = *static_cast<const typename Body::Args*>(a);
  flep_slice<Body><<<count, Body::kThreads, 0, static_cast<cudaStream_t>(s)>>>(
      args, g.x, g.y, offset, *static_cast<const SliceParams*>(sp));
  return static_cast<int>(cudaGetLastError());
}

template <class Body>
void user_body_ops(flep_body_ops* o, const char* name) {
  static_assert(!Body::kPersistent, "user bodies run original blocks (kPersistent = false)");
  o->abi_version = FLEP_BODY_ABI_VERSION;
  o->threads = static_cast<uint32_t>(Body::kThreads);
  o->args_size = sizeof(typename Body::Args);
  o->name = name;
  o->worker = &user_worker_launch<Body>;
  o->unwrapped = &user_unwrapped_launch<Body>;
  o->static_launch = &user_static_launch<Body>;
  o->occupancy = &user_occupancy<Body>;
  o->clc = &user_clc_launch<Body>;
  o->sliced = &user_slice_launch<Body>;
}

}  // namespace flep

#define FLEP_DEFINE_BODY(sym, Body) \
  extern "C" void sym##_ops(flep_body_ops* out) { flep::user_body_ops<Body>(out, #sym); }
