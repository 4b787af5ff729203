// keys.cuh -- order codes, (code, index) entries and the fast streaming predicate.
//
// The paper describes the method "for tuples consisting only of a key" and compares
// with `x0 < x1` (Alg. 4 line 9).  To make every compare-exchange a total order
// (bit-exact indices under ties, defined NaN / +-0; R1-R3) the networks
// compare ENTRIES: (order code, source index), better = larger code, then lower index.
//
//  * E32 -- 32-bit codes (f32, u32): one uint64 = code << 32 | ~lidx, so "better" is a
//    single unsigned 64-bit compare.  lidx is the row offset inside the launch
//    (< 2^32 - 1); ~lidx makes lower indices larger.  Sentinel (padding, "padded
//    with min/max value so that they never show up") = 0: code 0 with lidx 0xFFFFFFFF,
//    worse than every real key, including a real key of code 0.
//  * E64 -- 64-bit codes (f64): {code, ~lidx}; sentinel = {0, 0}.
#pragma once
#include <cstdint>

namespace topk {

struct E32 {
    uint64_t v;
    __device__ __forceinline__ static E32 make(uint32_t code, uint32_t lidx) {
        return E32{(static_cast<uint64_t>(code) << 32) | static_cast<uint32_t>(~lidx)};
    }
    __device__ __forceinline__ static E32 sentinel() { return E32{0ull}; }
    __device__ __forceinline__ bool is_sentinel() const { return v == 0ull; }
    __device__ __forceinline__ uint32_t lidx() const { return ~static_cast<uint32_t>(v); }
    __device__ __forceinline__ uint64_t code() const { return v >> 32; }
};
__device__ __forceinline__ bool better(E32 a, E32 b) { return a.v > b.v; }

struct E64 {
    uint64_t c;
    uint32_t ni;
    __device__ __forceinline__ static E64 make(uint64_t code, uint32_t lidx) {
        return E64{code, ~lidx};
    }
    __device__ __forceinline__ static E64 sentinel() { return E64{0ull, 0u}; }
    __device__ __forceinline__ bool is_sentinel() const { return c == 0ull && ni == 0u; }
    __device__ __forceinline__ uint32_t lidx() const { return ~ni; }
    __device__ __forceinline__ uint64_t code() const { return c; }
};
__device__ __forceinline__ bool better(E64 a, E64 b) {
    return a.c > b.c || (a.c == b.c && a.ni > b.ni);
}

// E96 -- three compound f32 keys (KKKV, R19): {c = code(k1) << 32 | code(k2),
// c3 = code(k3), ~lidx}, compared lexicographically; sentinel = {0, 0, 0}.
struct E96 {
    uint64_t c;
    uint32_t c3;
    uint32_t ni;
    __device__ __forceinline__ static E96 make(uint64_t code, uint32_t code3, uint32_t lidx) {
        return E96{code, code3, ~lidx};
    }
    __device__ __forceinline__ static E96 sentinel() { return E96{0ull, 0u, 0u}; }
    __device__ __forceinline__ bool is_sentinel() const { return c == 0ull && c3 == 0u && ni == 0u; }
    __device__ __forceinline__ uint32_t lidx() const { return ~ni; }
    __device__ __forceinline__ uint64_t code() const { return c; }
};
__device__ __forceinline__ bool better(E96 a, E96 b) {
    // (c3, ni) as one 64-bit word: c3 decides, then the lower row (larger ~lidx)
    const uint64_t la = (static_cast<uint64_t>(a.c3) << 32) | a.ni;
    const uint64_t lb = (static_cast<uint64_t>(b.c3) << 32) | b.ni;
    return a.c > b.c || (a.c == b.c && la > lb);
}

// Branch-free select (selp): the compiler otherwise turns data-dependent swaps into
// divergent branches, serialising the warp.
__device__ __forceinline__ uint64_t sel64(bool p, uint64_t a, uint64_t b) {
    uint64_t r;
    asm("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\tselp.b64 %0, %1, %2, q;\n\t}"
        : "=l"(r)
        : "l"(a), "l"(b), "r"(static_cast<uint32_t>(p)));
    return r;
}
__device__ __forceinline__ uint32_t sel32(bool p, uint32_t a, uint32_t b) {
    uint32_t r;
    asm("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\tselp.b32 %0, %1, %2, q;\n\t}"
        : "=r"(r)
        : "r"(a), "r"(b), "r"(static_cast<uint32_t>(p)));
    return r;
}
__device__ __forceinline__ E32 esel(bool p, E32 a, E32 b) { return E32{sel64(p, a.v, b.v)}; }
__device__ __forceinline__ E64 esel(bool p, E64 a, E64 b) {
    return E64{sel64(p, a.c, b.c), sel32(p, a.ni, b.ni)};
}
__device__ __forceinline__ E96 esel(bool p, E96 a, E96 b) {
    return E96{sel64(p, a.c, b.c), sel32(p, a.c3, b.c3), sel32(p, a.ni, b.ni)};
}

// Shared-memory arrays of entries (structure of arrays for E64: 12 B per entry).
// Entry index e is stored at swz(e) = e ^ (((e >> 4) & 7) << 1): the 16-byte column of
// a 128-byte row is XORed with the row number, so a warp whose lanes each read one
// 16-entry row (the register networks' blocked layout) hits 8 distinct columns per
// quarter-warp -- conflict-free (the B200 analogue of the paper's padding / chunk
// permutation).  Pairs (2j, 2j+1) stay adjacent (16-byte loads).
__device__ __forceinline__ int swz(int e) { return e ^ (((e >> 4) & 7) << 1); }

template <class E>
struct SBuf;
template <>
struct SBuf<E32> {
    uint64_t* v;
    static constexpr int kBytes = 8;
    __device__ __forceinline__ void init(unsigned char* base, int cap) {
        v = reinterpret_cast<uint64_t*>(base);
        (void)cap;
    }
    __device__ __forceinline__ E32 ld(int i) const { return E32{v[swz(i)]}; }
    __device__ __forceinline__ void st(int i, E32 e) const { v[swz(i)] = e.v; }
    // entries i, i+1 (i even) with one 16-byte access
    __device__ __forceinline__ void ld2(int i, E32& a, E32& b) const {
        const ulonglong2 q = *reinterpret_cast<const ulonglong2*>(v + swz(i));
        a = E32{q.x};
        b = E32{q.y};
    }
    __device__ __forceinline__ void st2(int i, E32 a, E32 b) const {
        *reinterpret_cast<ulonglong2*>(v + swz(i)) = make_ulonglong2(a.v, b.v);
    }
};
template <>
struct SBuf<E64> {
    uint64_t* c;
    uint32_t* ni;
    static constexpr int kBytes = 12;
    __device__ __forceinline__ void init(unsigned char* base, int cap) {
        c = reinterpret_cast<uint64_t*>(base);
        ni = reinterpret_cast<uint32_t*>(base + 8 * static_cast<size_t>(cap));
    }
    __device__ __forceinline__ E64 ld(int i) const {
        const int j = swz(i);
        return E64{c[j], ni[j]};
    }
    __device__ __forceinline__ void st(int i, E64 e) const {
        const int j = swz(i);
        c[j] = e.c;
        ni[j] = e.ni;
    }
    __device__ __forceinline__ void ld2(int i, E64& a, E64& b) const {
        const int j = swz(i);
        const ulonglong2 q = *reinterpret_cast<const ulonglong2*>(c + j);
        const uint2 n = *reinterpret_cast<const uint2*>(ni + j);
        a = E64{q.x, n.x};
        b = E64{q.y, n.y};
    }
    __device__ __forceinline__ void st2(int i, E64 a, E64 b) const {
        const int j = swz(i);
        *reinterpret_cast<ulonglong2*>(c + j) = make_ulonglong2(a.c, b.c);
        *reinterpret_cast<uint2*>(ni + j) = make_uint2(a.ni, b.ni);
    }
};

template <>
struct SBuf<E96> {
    uint64_t* c;
    uint32_t* c3;
    uint32_t* ni;
    static constexpr int kBytes = 16;
    __device__ __forceinline__ void init(unsigned char* base, int cap) {
        c = reinterpret_cast<uint64_t*>(base);
        c3 = reinterpret_cast<uint32_t*>(base + 8 * static_cast<size_t>(cap));
        ni = reinterpret_cast<uint32_t*>(base + 12 * static_cast<size_t>(cap));
    }
    __device__ __forceinline__ E96 ld(int i) const {
        const int j = swz(i);
        return E96{c[j], c3[j], ni[j]};
    }
    __device__ __forceinline__ void st(int i, E96 e) const {
        const int j = swz(i);
        c[j] = e.c;
        c3[j] = e.c3;
        ni[j] = e.ni;
    }
    __device__ __forceinline__ void ld2(int i, E96& a, E96& b) const {
        const int j = swz(i);
        const ulonglong2 q = *reinterpret_cast<const ulonglong2*>(c + j);
        const uint2 t = *reinterpret_cast<const uint2*>(c3 + j);
        const uint2 n = *reinterpret_cast<const uint2*>(ni + j);
        a = E96{q.x, t.x, n.x};
        b = E96{q.y, t.y, n.y};
    }
    __device__ __forceinline__ void st2(int i, E96 a, E96 b) const {
        const int j = swz(i);
        *reinterpret_cast<ulonglong2*>(c + j) = make_ulonglong2(a.c, b.c);
        *reinterpret_cast<uint2*>(c3 + j) = make_uint2(a.c3, b.c3);
        *reinterpret_cast<uint2*>(ni + j) = make_uint2(a.ni, b.ni);
    }
};

// ---------------------------------------------------------------------------------
// Key traits: code(), threshold decode and the streaming fast test.
//
// code_max(x): order-preserving unsigned image (R2).  IEEE-754 patterns of
// non-negative numbers grow with the value -> set the top bit; negative patterns
// shrink -> complement.  Overrides: every NaN -> all ones (ranks above +inf, all NaNs
// tie); -0 -> the code of +0.  Min order uses ~code_max(x).
//
// fast<MIN, STRICT>(x, t): a superset test "x may beat the threshold key t", used on
// every streamed key (1 FSETP/ISETP per key).  For floats the unordered variants
// (GTU/GEU/LTU/LEU) keep NaN keys, which the exact entry test then decides.
// ---------------------------------------------------------------------------------
template <class K>
struct KeyTraits;

template <>
struct KeyTraits<float> {
    using Key = float;
    using E = E32;
    using Vec = float4;
    static constexpr int kVec = 4;
    __device__ __forceinline__ static uint32_t code_max(float x) {
        uint32_t u = __float_as_uint(x);
        uint32_t c = (u & 0x80000000u) ? ~u : (u | 0x80000000u);
        if (x == 0.0f) c = 0x80000000u;
        if (x != x) c = 0xFFFFFFFFu;
        return c;
    }
    template <bool MIN>
    __device__ __forceinline__ static uint32_t code(float x) {
        return MIN ? ~code_max(x) : code_max(x);
    }
    // A key whose code equals `c` (NaN if c is the NaN code).
    template <bool MIN>
    __device__ __forceinline__ static float decode(uint64_t c64) {
        uint32_t c = static_cast<uint32_t>(c64);
        if (MIN) c = ~c;
        if (c == 0xFFFFFFFFu) return __uint_as_float(0x7FC00000u);
        uint32_t u = (c & 0x80000000u) ? (c & 0x7FFFFFFFu) : ~c;
        return __uint_as_float(u);
    }
    template <bool MIN, bool STRICT>
    __device__ __forceinline__ static bool fast(float x, float t) {
        if (MIN) return STRICT ? !(x >= t) : !(x > t);
        return STRICT ? !(x <= t) : !(x < t);
    }
};

template <>
struct KeyTraits<uint32_t> {
    using Key = uint32_t;
    using E = E32;
    using Vec = uint4;
    static constexpr int kVec = 4;
    template <bool MIN>
    __device__ __forceinline__ static uint32_t code(uint32_t x) {
        return MIN ? ~x : x;
    }
    template <bool MIN>
    __device__ __forceinline__ static uint32_t decode(uint64_t c64) {
        uint32_t c = static_cast<uint32_t>(c64);
        return MIN ? ~c : c;
    }
    template <bool MIN, bool STRICT>
    __device__ __forceinline__ static bool fast(uint32_t x, uint32_t t) {
        if (MIN) return STRICT ? (x < t) : (x <= t);
        return STRICT ? (x > t) : (x >= t);
    }
};

template <>
struct KeyTraits<double> {
    using Key = double;
    using E = E64;
    using Vec = double2;
    static constexpr int kVec = 2;
    __device__ __forceinline__ static uint64_t code_max(double x) {
        uint64_t u = static_cast<uint64_t>(__double_as_longlong(x));
        uint64_t c = (u >> 63) ? ~u : (u | 0x8000000000000000ull);
        if (x == 0.0) c = 0x8000000000000000ull;
        if (x != x) c = ~0ull;
        return c;
    }
    template <bool MIN>
    __device__ __forceinline__ static uint64_t code(double x) {
        return MIN ? ~code_max(x) : code_max(x);
    }
    template <bool MIN>
    __device__ __forceinline__ static double decode(uint64_t c) {
        if (MIN) c = ~c;
        if (c == ~0ull) return __longlong_as_double(0x7FF8000000000000ll);
        uint64_t u = (c >> 63) ? (c & 0x7FFFFFFFFFFFFFFFull) : ~c;
        return __longlong_as_double(static_cast<long long>(u));
    }
    template <bool MIN, bool STRICT>
    __device__ __forceinline__ static bool fast(double x, double t) {
        if (MIN) return STRICT ? !(x >= t) : !(x > t);
        return STRICT ? !(x <= t) : !(x < t);
    }
};

// Compound key (two f32 columns a, b, ORDER BY a, b -- KKV; R19):
// a tag type for the select kernel's query form kQKey2.  The entry is E64 with the
// 64-bit code (code(a) << 32) | code2(b): one unsigned compare is the lexicographic
// order, the row id breaks the remaining ties.  The streamed a column is read as
// float4 like f32 keys; the kernel computes codes directly (no threshold key).
struct KK32 {
    float a;
};
template <>
struct KeyTraits<KK32> {
    using Key = KK32;
    using E = E64;
    using Vec = float4;
    static constexpr int kVec = 4;
    template <bool MIN>
    __device__ __forceinline__ static KK32 decode(uint64_t) {
        return KK32{0.f};  // unused: the compound fast test compares codes
    }
    // (code(a) << 32) | code(b): a in the kernel's order, b in order2 (1 = ascending)
    template <bool MIN>
    __device__ __forceinline__ static uint64_t code2(float a, float b, uint32_t b_min) {
        const uint32_t cb = KeyTraits<float>::code_max(b);
        return (static_cast<uint64_t>(KeyTraits<float>::code<MIN>(a)) << 32) | (b_min ? ~cb : cb);
    }
};

// Three compound keys (a, b, c; KKKV): tag type of the select kernel's query form
// kQKey2 | kQKey3, entry E96.
struct KKK32 {
    float a;
};
template <>
struct KeyTraits<KKK32> {
    using Key = KKK32;
    using E = E96;
    using Vec = float4;
    static constexpr int kVec = 4;
    template <bool MIN>
    __device__ __forceinline__ static KKK32 decode(uint64_t) {
        return KKK32{0.f};  // unused: the compound fast test compares codes
    }
    template <bool MIN>
    __device__ __forceinline__ static uint64_t code2(float a, float b, uint32_t b_min) {
        return KeyTraits<KK32>::code2<MIN>(a, b, b_min);
    }
    __device__ __forceinline__ static uint32_t code3(float c, uint32_t c_min) {
        const uint32_t cc = KeyTraits<float>::code_max(c);
        return c_min ? ~cc : cc;
    }
};

}  // namespace topk
