// dispatch.cuh -- runtime (dtype, op, map) -> template instantiation.
#pragma once
#include <type_traits>

#include "common.cuh"

namespace ifl {

template <int V>
using IC = std::integral_constant<int, V>;

template <typename T, int F, typename Fn>
cudaError_t dispatch_op(int op, Fn&& fn) {
    switch (op) {
    case OP_SUM: return fn(T{}, IC<OP_SUM>{}, IC<F>{});
    case OP_PROD: return fn(T{}, IC<OP_PROD>{}, IC<F>{});
    case OP_MIN: return fn(T{}, IC<OP_MIN>{}, IC<F>{});
    case OP_MAX: return fn(T{}, IC<OP_MAX>{}, IC<F>{});
    default: break;
    }
    if constexpr (std::is_same<T, int>::value) {
        switch (op) {
        case OP_AND: return fn(T{}, IC<OP_AND>{}, IC<F>{});
        case OP_OR: return fn(T{}, IC<OP_OR>{}, IC<F>{});
        case OP_XOR: return fn(T{}, IC<OP_XOR>{}, IC<F>{});
        default: break;
        }
    }
    return cudaErrorInvalidValue;
}

template <typename T, typename Fn>
cudaError_t dispatch_map(int op, int f, Fn&& fn) {
    switch (f) {
    case F_ID: return dispatch_op<T, F_ID>(op, fn);
    case F_SQ: return dispatch_op<T, F_SQ>(op, fn);
    case F_ABS: return dispatch_op<T, F_ABS>(op, fn);
    default: return cudaErrorInvalidValue;
    }
}

// dt: 0 = int32, 1 = float32 (ifl_dtype)
template <typename Fn>
cudaError_t dispatch_all(int dt, int op, int f, Fn&& fn) {
    if (dt == 0) return dispatch_map<int>(op, f, fn);
    if (dt == 1) return dispatch_map<float>(op, f, fn);
    return cudaErrorInvalidValue;
}

template <typename T>
__host__ inline T bits_to(uint32_t u) {
    T v;
    static_assert(sizeof(T) == 4, "32-bit element types only");
    memcpy(&v, &u, 4);
    return v;
}

}  // namespace ifl
