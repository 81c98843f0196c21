"""Small wrapped launches for compute-sanitizer (memcheck / racecheck / synccheck): every body,
one temporal and one spatial preemption with resume, the CLC task fetch (with a preempt/resume
cycle), the TMA-staged stencil (counter and CLC workers, chunk 2 so the second input buffer is
used) and in-tile GEMM preemption."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import gen  # noqa: E402


def main():
    import torch
    from paper_conf_asplos_wulzj17_b200 import build, flep as F
    build.build()
    T = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
    rt = F.Runtime(coverage=True)
    n = 1 << 14
    x, y = gen.saxpy_i32_inputs(n, 1)
    xd, yd = T(x), T(y)
    k = rt.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1, ctas_per_sm=1)
    for nsm in (rt.num_sms, 8):
        rt.arm_next_trigger(n // 512, nsm)
        h = rt.launch(k, F.saxpy_grid(n), F.saxpy_i32_args(yd, xd, 3))
        rt.wait_epoch(h)
        if rt.query(h).state == F.STATE_PREEMPTED:
            rt.resume(h)
        rt.sync(h)
    rp, col, val, xv = gen.csr_inputs(2000, 2)
    yv = torch.zeros(2000, device="cuda")
    k2 = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=2, poll=1, prefetch=True)
    keep = (T(rp), T(col), T(val), T(xv))       # outlive the args struct (raw pointers)
    rt.sync(rt.launch(k2, F.spmv_grid(2000), F.spmv_args(yv, *keep)))
    st = T(gen.stencil_f32_input(200, 3))
    out = torch.empty_like(st)
    k3 = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=1)
    rt.sync(rt.launch(k3, F.stencil_grid(200), F.stencil_args(out, st)))
    a_bits, b_bits = gen.gemm_bf16_inputs(256, 512, 128, 4)
    A = torch.from_numpy(a_bits.view(np.int16)).cuda().view(torch.bfloat16)
    B = torch.from_numpy(b_bits.view(np.int16)).cuda().view(torch.bfloat16)
    C = torch.empty(256, 512, dtype=torch.bfloat16, device="cuda")
    k4 = rt.register_kernel(F.BODY_GEMM_BF16, chunk=1, poll=1)
    rt.sync(rt.launch(k4, F.gemm_grid(256, 512), F.gemm_args(C, A, B)))
    # request-relay CTA (R28): a host preempt/resume cycle through the relay
    k8 = rt.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1, host_relay=True)
    h = rt.launch(k8, F.saxpy_grid(n), F.saxpy_i32_args(yd, xd, 9))
    try:
        rt.preempt(h, rt.num_sms)
        rt.wait_epoch(h)
        if rt.query(h).state == F.STATE_PREEMPTED:
            rt.resume(h)
    except F.FlepError:
        pass
    rt.sync(h)
    # CLC task fetch: uninterrupted, then a host preempt/resume cycle
    k5 = rt.register_kernel(F.BODY_SAXPY_I32, chunk=2, poll=1, clc=True)
    rt.sync(rt.launch(k5, F.saxpy_grid(n), F.saxpy_i32_args(yd, xd, 5)))
    h = rt.launch(k5, F.saxpy_grid(n), F.saxpy_i32_args(yd, xd, 7))
    try:
        rt.preempt(h, rt.num_sms)
        rt.resume(h)
    except F.FlepError:
        pass                              # completed first
    rt.sync(h)
    # TMA-staged stencil: unwrapped, counter worker and CLC worker (chunk 2: double buffer)
    st2 = T(gen.stencil_f32_input(260, 5))
    out2 = torch.empty_like(st2)
    rt.launch_unwrapped(F.BODY_STENCIL5_F32_TMA, F.stencil_grid(260), F.stencil_args(out2, st2))
    for clc in (False, True):
        k6 = rt.register_kernel(F.BODY_STENCIL5_F32_TMA, chunk=2, poll=1, clc=clc)
        rt.sync(rt.launch(k6, F.stencil_grid(260), F.stencil_args(out2, st2)))
    # in-tile GEMM preemption with resume
    a_bits, b_bits = gen.gemm_bf16_inputs(256, 512, 1024, 6)
    A = torch.from_numpy(a_bits.view(np.int16)).cuda().view(torch.bfloat16)
    B = torch.from_numpy(b_bits.view(np.int16)).cuda().view(torch.bfloat16)
    C = torch.empty(256, 512, dtype=torch.bfloat16, device="cuda")
    k7 = rt.register_kernel(F.BODY_GEMM_BF16, chunk=1, poll=1, ctas_per_sm=1, in_tile=True)
    rt.arm_next_trigger(1, rt.num_sms)
    h = rt.launch(k7, F.gemm_grid(256, 512), F.gemm_args(C, A, B))
    rt.wait_epoch(h)
    if rt.query(h).state == F.STATE_PREEMPTED:
        rt.resume(h)
    rt.sync(h)
    # round 2: warp-task workers (SpMV vector body, stencil) with a temporal preempt/resume cycle,
    # the static persistent twin, the CTA-pair GEMM (unwrapped, static, worker with a preemption, in-tile worker)
    # device-checked slicing with a preemption and the speculative fetch with a preemption
    k9 = rt.register_kernel(F.BODY_SPMV_CSR_F32_VEC, chunk=2, poll=1, warp_tasks=True)
    rt.arm_next_trigger(4, rt.num_sms)
    h = rt.launch(k9, F.spmv_grid(2000), F.spmv_args(yv, *keep))
    rt.wait_epoch(h)
    if rt.query(h).state == F.STATE_PREEMPTED:
        rt.resume(h)
    rt.sync(h)
    k10 = rt.register_kernel(F.BODY_STENCIL5_F32, chunk=1, poll=1, warp_tasks=True)
    rt.sync(rt.launch(k10, F.stencil_grid(200), F.stencil_args(out, st)))
    rt.launch_static(F.BODY_SPMV_CSR_F32, F.spmv_grid(2000), F.spmv_args(yv, *keep), chunk=2)
    a_bits, b_bits = gen.gemm_bf16_inputs(512, 512, 256, 8)
    A2 = torch.from_numpy(a_bits.view(np.int16)).cuda().view(torch.bfloat16)
    B2 = torch.from_numpy(b_bits.view(np.int16)).cuda().view(torch.bfloat16)
    C2 = torch.empty(512, 512, dtype=torch.bfloat16, device="cuda")
    g2 = F.gemm2_grid(512, 512)
    rt.launch_unwrapped(F.BODY_GEMM_BF16_2SM, g2, F.gemm_args(C2, A2, B2))
    rt.launch_static(F.BODY_GEMM_BF16_2SM, g2, F.gemm_args(C2, A2, B2))
    k11 = rt.register_kernel(F.BODY_GEMM_BF16_2SM, chunk=1, poll=1)
    rt.arm_next_trigger(1, rt.num_sms)
    h = rt.launch(k11, g2, F.gemm_args(C2, A2, B2))
    rt.wait_epoch(h)
    if rt.query(h).state == F.STATE_PREEMPTED:
        rt.resume(h)
    rt.sync(h)
    # speculative fetch (R34): a preempt/resume cycle that returns fetched chunks through records
    k13 = rt.register_kernel(F.BODY_SPMV_CSR_F32, chunk=1, poll=1, spec_fetch=True)
    rt.arm_next_trigger(4, rt.num_sms)
    h = rt.launch(k13, F.spmv_grid(2000), F.spmv_args(yv, *keep))
    rt.wait_epoch(h)
    if rt.query(h).state == F.STATE_PREEMPTED:
        rt.resume(h)
    rt.sync(h)
    k12 = rt.register_kernel(F.BODY_GEMM_BF16_2SM, chunk=1, poll=1, in_tile=True)
    a_bits, b_bits = gen.gemm_bf16_inputs(512, 512, 1024, 9)
    A3 = torch.from_numpy(a_bits.view(np.int16)).cuda().view(torch.bfloat16)
    B3 = torch.from_numpy(b_bits.view(np.int16)).cuda().view(torch.bfloat16)
    C3 = torch.empty(512, 512, dtype=torch.bfloat16, device="cuda")
    rt.arm_next_trigger(1, rt.num_sms)
    h = rt.launch(k12, g2, F.gemm_args(C3, A3, B3))
    rt.wait_epoch(h)
    if rt.query(h).state == F.STATE_PREEMPTED:
        rt.resume(h)
    rt.sync(h)
    # the wide pair tile (256x512): unwrapped, static, worker preempted tile-granular and in-tile
    a_bits, b_bits = gen.gemm_bf16_inputs(512, 1024, 1024, 10)
    A4 = torch.from_numpy(a_bits.view(np.int16)).cuda().view(torch.bfloat16)
    B4 = torch.from_numpy(b_bits.view(np.int16)).cuda().view(torch.bfloat16)
    C4 = torch.empty(512, 1024, dtype=torch.bfloat16, device="cuda")
    g2w = F.gemm2w_grid(512, 1024)
    rt.launch_unwrapped(F.BODY_GEMM_BF16_2SM_W, g2w, F.gemm_args(C4, A4, B4))
    rt.launch_static(F.BODY_GEMM_BF16_2SM_W, g2w, F.gemm_args(C4, A4, B4))
    for in_tile in (False, True):
        k14 = rt.register_kernel(F.BODY_GEMM_BF16_2SM_W, chunk=1, poll=1, in_tile=in_tile)
        rt.arm_next_trigger(1, rt.num_sms)
        h = rt.launch(k14, g2w, F.gemm_args(C4, A4, B4))
        rt.wait_epoch(h)
        if rt.query(h).state == F.STATE_PREEMPTED:
            rt.resume(h)
        rt.sync(h)
    torch.cuda.synchronize()
    rt.close()
    rs = F.Runtime(policy=F.POLICY_SLICE_DEVICE, slice_blocks=8)
    kl = rs.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 1_000_000))
    kh = rs.register_kernel(F.BODY_SAXPY_I32, chunk=1, poll=1, model=(0, 0, 0, 0, 1_000))
    x3, y3 = gen.saxpy_i32_inputs(256, 3)
    x3d, y3d = T(x3), T(y3)
    h1 = rs.launch(kl, F.saxpy_grid(n), F.saxpy_i32_args(yd, xd, 3), priority=0)
    h2 = rs.launch(kh, F.saxpy_grid(256), F.saxpy_i32_args(y3d, x3d, 5), priority=1)
    rs.sync(h2)
    rs.sync(h1)
    torch.cuda.synchronize()
    rs.close()
    print("sanitizer case done")


if __name__ == "__main__":
    main()
