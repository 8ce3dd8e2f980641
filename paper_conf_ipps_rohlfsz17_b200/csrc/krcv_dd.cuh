// krcv_dd.cuh -- double-double ("dd") arithmetic for the window-prefix path.
//
// A dd value is hi + lo with |lo| <= ulp(hi)/2: ~106 significant bits from
// two binary64 numbers.  The window-prefix path (krcv_prefix.cuh) keeps the
// prefix sums of the moments y, u, u^2, y u, y u^2 (u = x - origin) in dd so
// that a window's sums, P[R] - P[L+1], and their shift to the row's own
// origin, sum (u - delta)^2 = Suu - delta (2 Su - c delta), lose nothing
// to cancellation at the 1e-16 level (DESIGN.md §6.2 gives the error bound).
//
// Error-free transformations (Knuth two-sum, FMA two-product).  Every
// operation uses the __d*_rn intrinsics so nvcc can neither contract a
// product into an FMA nor otherwise change the rounding the algorithms rely on.
#pragma once

#include <cuda_runtime.h>

namespace krcv {

struct dd {
    double hi, lo;
};

__device__ __forceinline__ dd dd_make(double a) { return dd{a, 0.0}; }

// s + e == a + b exactly (no magnitude precondition).  6 FP64 ops.
__device__ __forceinline__ dd two_sum(double a, double b)
{
    const double s = __dadd_rn(a, b);
    const double bb = __dsub_rn(s, a);
    const double e = __dadd_rn(__dsub_rn(a, __dsub_rn(s, bb)), __dsub_rn(b, bb));
    return dd{s, e};
}

// s + e == a + b exactly, requires |a| >= |b| (or a == 0).  3 FP64 ops.
__device__ __forceinline__ dd quick_two_sum(double a, double b)
{
    const double s = __dadd_rn(a, b);
    const double e = __dsub_rn(b, __dsub_rn(s, a));
    return dd{s, e};
}

// p + e == a * b exactly.  2 FP64 ops.
__device__ __forceinline__ dd two_prod(double a, double b)
{
    const double p = __dmul_rn(a, b);
    const double e = __fma_rn(a, b, -p);
    return dd{p, e};
}

// a + b.  Absolute error <= ~2 eps^2 max(|a|, |b|) ("sloppy" add: enough for
// differences of prefix sums, where the absolute error is what matters).
__device__ __forceinline__ dd dd_add(dd a, dd b)
{
    dd s = two_sum(a.hi, b.hi);
    s.lo = __dadd_rn(s.lo, __dadd_rn(a.lo, b.lo));
    return quick_two_sum(s.hi, s.lo);
}

__device__ __forceinline__ dd dd_neg(dd a) { return dd{-a.hi, -a.lo}; }

__device__ __forceinline__ dd dd_sub(dd a, dd b) { return dd_add(a, dd_neg(b)); }

// a + b with b a double.
__device__ __forceinline__ dd dd_add_d(dd a, double b)
{
    dd s = two_sum(a.hi, b);
    s.lo = __dadd_rn(s.lo, a.lo);
    return quick_two_sum(s.hi, s.lo);
}

// a * b with b a double.
__device__ __forceinline__ dd dd_mul_d(dd a, double b)
{
    dd p = two_prod(a.hi, b);
    p.lo = __fma_rn(a.lo, b, p.lo);
    return quick_two_sum(p.hi, p.lo);
}

// a * b (drops lo*lo, ~2^-104 relative).
__device__ __forceinline__ dd dd_mul(dd a, dd b)
{
    dd p = two_prod(a.hi, b.hi);
    p.lo = __fma_rn(a.hi, b.lo, __fma_rn(a.lo, b.hi, p.lo));
    return quick_two_sum(p.hi, p.lo);
}

// a * b and a * (double) b without the final renormalisation: |lo| stays
// O(eps |hi|), which every consumer below (dd_add / dd_sub_to_d) accepts.
__device__ __forceinline__ dd dd_mul_raw(dd a, dd b)
{
    dd p = two_prod(a.hi, b.hi);
    p.lo = __fma_rn(a.hi, b.lo, __fma_rn(a.lo, b.hi, p.lo));
    return p;
}

__device__ __forceinline__ dd dd_mul_d_raw(dd a, double b)
{
    dd p = two_prod(a.hi, b);
    p.lo = __fma_rn(a.lo, b, p.lo);
    return p;
}

// a - b rounded to the nearest double (within 1 ulp): the last step of a
// dd computation whose result is consumed in double.
__device__ __forceinline__ double dd_sub_to_d(dd a, dd b)
{
    const dd s = two_sum(a.hi, -b.hi);
    return __dadd_rn(s.hi, __dadd_rn(s.lo, __dsub_rn(a.lo, b.lo)));
}

// 2^k scaling is exact.
__device__ __forceinline__ dd dd_twice(dd a) { return dd{__dmul_rn(2.0, a.hi), __dmul_rn(2.0, a.lo)}; }

// Nearest double (hi already is, up to the renormalisation above).
__device__ __forceinline__ double dd_to_d(dd a) { return __dadd_rn(a.hi, a.lo); }

}  // namespace krcv
