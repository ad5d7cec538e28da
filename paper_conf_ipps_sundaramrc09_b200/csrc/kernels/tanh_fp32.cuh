// tanh_fp32.cuh -- tanh for the fp32 paths (TG_FP32, TG_FP32_TC, the operator library).
//
// PAPER.md:635 (torch5 Tanh; R9). The fp32 parity bound (1e-5 normwise, R16) is
// set by the arithmetic around the tanh layers, so tanh itself must be accurate to a few
// fp32 ulps RELATIVE to its result, also near 0:
//   |x| <  0.6: tanh x = x + x s q(s), s = x^2, q a degree-4 minimax fit of (tanh x / x - 1)/s
//               on [0, 0.36] (fit error 2.8e-9 relative; 1.2 ulp max evaluated in fp32);
//   |x| >= 0.6: sign(x) (1 - 2 / (1 + e^{2|x|})) from MUFU ex2 and rcp (|tanh| >= 0.537, so the
//               subtraction loses nothing; e^{2|x|} -> inf gives exactly 1).
// The earlier one-branch 1 - 2/(1+e^{2x}) had an ABSOLUTE error of ~2e-7 near 0 (the
// subtraction cancels): the dominant error of both fp32 CNN paths.
#pragma once

namespace tg {

__device__ __forceinline__ float tanh_fp32(float x) {
    const float ax = fabsf(x);
    float e, r;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e) : "f"(ax * 2.885390081777927f));  // 2 log2(e) |x|
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(1.f + e));
    const float big = copysignf(fmaf(-2.f, r, 1.f), x);
    const float s = x * x;
    float q = fmaf(-0.005895121023058891f, s, 0.02079593949019909f);
    q = fmaf(q, s, -0.05378381907939911f);
    q = fmaf(q, s, 0.13331924378871918f);
    q = fmaf(q, s, -0.33333298563957214f);
    const float small = fmaf(x * s, q, x);
    return ax < 0.6f ? small : big;
}

// The same function on a pair, with the FMA-pipe arithmetic as paired FP32 instructions (FFMA2 /
// FMUL2 / FADD2, sm_100): each lane rounds exactly like the scalar fmaf / fmul / fadd, so the
// result is bit-identical to tanh_fp32 on each element, for about half the FMA-pipe issue slots.
__device__ __forceinline__ float2 tanh_fp32x2(float2 x) {
    const float2 ax = make_float2(fabsf(x.x), fabsf(x.y));
    const float2 arg = __fmul2_rn(ax, make_float2(2.885390081777927f, 2.885390081777927f));
    float2 e, r;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e.x) : "f"(arg.x));
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e.y) : "f"(arg.y));
    const float2 d = __fadd2_rn(make_float2(1.f, 1.f), e);
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r.x) : "f"(d.x));
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r.y) : "f"(d.y));
    const float2 m = __ffma2_rn(make_float2(-2.f, -2.f), r, make_float2(1.f, 1.f));
    const float2 s = __fmul2_rn(x, x);
    float2 q = __ffma2_rn(make_float2(-0.005895121023058891f, -0.005895121023058891f), s,
                          make_float2(0.02079593949019909f, 0.02079593949019909f));
    q = __ffma2_rn(q, s, make_float2(-0.05378381907939911f, -0.05378381907939911f));
    q = __ffma2_rn(q, s, make_float2(0.13331924378871918f, 0.13331924378871918f));
    q = __ffma2_rn(q, s, make_float2(-0.33333298563957214f, -0.33333298563957214f));
    const float2 small = __ffma2_rn(__fmul2_rn(x, s), q, x);
    return make_float2(ax.x < 0.6f ? small.x : copysignf(m.x, x.x), ax.y < 0.6f ? small.y : copysignf(m.y, x.y));
}

}  // namespace tg
