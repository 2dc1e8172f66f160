// hbig.h -- small host-side unsigned big integer in binary limbs (product code).
//
// Used only at query-compile time: literal constants, 10^k alignment
// multipliers, 10^p overflow bounds, Montgomery constants for modexp, and
// formatting of final results.  Constants are converted once on the host and
// baked into generated kernels (§III-D2: "we migrate the
// constant conversion to the compilation from runtime execution").
#pragma once
#include <algorithm>
#include <cstdint>
#include <string>
#include <mutex>
#include <vector>

namespace uph {

struct HBig {
    std::vector<uint32_t> w;   // little-endian, trimmed (empty = 0)

    HBig() {}
    explicit HBig(uint64_t v) {
        while (v) { w.push_back((uint32_t)v); v >>= 32; }
    }
    void trim() { while (!w.empty() && w.back() == 0) w.pop_back(); }
    bool is_zero() const { return w.empty(); }
    int bitlen() const {
        if (w.empty()) return 0;
        return 32 * (int)(w.size() - 1) + (32 - __builtin_clz(w.back()));
    }
    uint32_t limb(size_t i) const { return i < w.size() ? w[i] : 0u; }
    bool bit(int i) const { return (limb((size_t)i / 32) >> (i % 32)) & 1u; }

    static int cmp(const HBig &a, const HBig &b) {
        if (a.w.size() != b.w.size()) return a.w.size() < b.w.size() ? -1 : 1;
        for (size_t i = a.w.size(); i-- > 0;)
            if (a.w[i] != b.w[i]) return a.w[i] < b.w[i] ? -1 : 1;
        return 0;
    }
    HBig mul_small(uint32_t m) const {
        HBig r; uint64_t c = 0;
        for (uint32_t x : w) { uint64_t t = (uint64_t)x * m + c; r.w.push_back((uint32_t)t); c = t >> 32; }
        if (c) r.w.push_back((uint32_t)c);
        r.trim(); return r;
    }
    HBig add_small(uint32_t a) const {
        HBig r = *this; uint64_t c = a;
        for (size_t i = 0; c && i < r.w.size(); ++i) { uint64_t t = (uint64_t)r.w[i] + c; r.w[i] = (uint32_t)t; c = t >> 32; }
        if (c) r.w.push_back((uint32_t)c);
        return r;
    }
    static HBig add(const HBig &a, const HBig &b) {
        HBig r; size_t n = std::max(a.w.size(), b.w.size()); uint64_t c = 0;
        for (size_t i = 0; i < n; ++i) { uint64_t t = (uint64_t)a.limb(i) + b.limb(i) + c; r.w.push_back((uint32_t)t); c = t >> 32; }
        if (c) r.w.push_back((uint32_t)c);
        r.trim(); return r;
    }
    static HBig sub(const HBig &a, const HBig &b) {   // requires a >= b
        HBig r; int64_t br = 0;
        for (size_t i = 0; i < a.w.size(); ++i) {
            int64_t t = (int64_t)a.w[i] - (int64_t)b.limb(i) - br;
            br = t < 0; if (t < 0) t += ((int64_t)1 << 32);
            r.w.push_back((uint32_t)t);
        }
        r.trim(); return r;
    }
    static HBig mul(const HBig &a, const HBig &b) {
        if (a.is_zero() || b.is_zero()) return HBig();
        HBig r; r.w.assign(a.w.size() + b.w.size(), 0);
        for (size_t i = 0; i < a.w.size(); ++i) {
            uint64_t c = 0;
            for (size_t j = 0; j < b.w.size(); ++j) {
                uint64_t t = (uint64_t)a.w[i] * b.w[j] + r.w[i + j] + c;
                r.w[i + j] = (uint32_t)t; c = t >> 32;
            }
            r.w[i + b.w.size()] = (uint32_t)c;
        }
        r.trim(); return r;
    }
    HBig shl1() const {
        HBig r; uint32_t c = 0;
        for (uint32_t x : w) { r.w.push_back((x << 1) | c); c = x >> 31; }
        if (c) r.w.push_back(c);
        return r;
    }
    HBig shl_limbs(int k) const {
        if (is_zero()) return HBig();
        HBig r; r.w.assign((size_t)k, 0); r.w.insert(r.w.end(), w.begin(), w.end()); return r;
    }
    // a mod m by binary shift-and-subtract (compile-time constants only)
    static HBig mod(const HBig &a, const HBig &m) {
        HBig r;
        for (int i = a.bitlen() - 1; i >= 0; --i) {
            r = r.shl1();
            if (a.bit(i)) r = r.add_small(1);
            if (cmp(r, m) >= 0) r = sub(r, m);
        }
        return r;
    }
    // divide by small d, returns remainder
    HBig div_small(uint32_t d, uint32_t &rem) const {
        HBig q; q.w.assign(w.size(), 0); uint64_t r = 0;
        for (size_t i = w.size(); i-- > 0;) { uint64_t t = (r << 32) | w[i]; q.w[i] = (uint32_t)(t / d); r = t % d; }
        q.trim(); rem = (uint32_t)r; return q;
    }
    // 10^k, memoised (typing and codegen ask for the same powers on every call;
    // recomputing 10^2000 digit by digit costs milliseconds of host time)
    static HBig pow10(int k) {
        static std::mutex mu;
        static std::vector<HBig> memo;
        std::lock_guard<std::mutex> g(mu);
        if (memo.empty()) memo.push_back(HBig(1));
        while ((int)memo.size() <= k) memo.push_back(memo.back().mul_small(10));
        return memo[(size_t)k];
    }
    // parse decimal digits (no sign, no point); returns false on a bad char
    static bool from_dec(const std::string &s, HBig &out) {
        HBig r;
        if (s.empty()) return false;
        for (char c : s) {
            if (c < '0' || c > '9') return false;
            r = r.mul_small(10).add_small((uint32_t)(c - '0'));
        }
        out = r; return true;
    }
    std::string to_dec() const {
        if (is_zero()) return "0";
        std::vector<uint32_t> parts; HBig t = *this;
        while (!t.is_zero()) { uint32_t rem; t = t.div_small(1000000000u, rem); parts.push_back(rem); }
        std::string s = std::to_string(parts.back());
        char buf[16];
        for (size_t i = parts.size() - 1; i-- > 0;) { snprintf(buf, sizeof buf, "%09u", parts[i]); s += buf; }
        return s;
    }
    int dec_digits() const { return is_zero() ? 1 : (int)to_dec().size(); }
    // two's complement limbs of (neg ? -x : x) in L limbs
    std::vector<uint32_t> twos(int L, bool neg) const {
        std::vector<uint32_t> r((size_t)L, 0);
        for (int i = 0; i < L; ++i) r[(size_t)i] = limb((size_t)i);
        if (neg) {
            uint64_t c = 1;
            for (int i = 0; i < L; ++i) { uint64_t t = (uint64_t)(~r[(size_t)i]) + c; r[(size_t)i] = (uint32_t)t; c = t >> 32; }
        }
        return r;
    }
};

// min L with 10^p <= 2^(32L-1)  (reproduces P:L1569-1575)
inline int limbs_for_precision(int p) {
    if (p <= 0) return 1;
    // 10^p is not a power of two for p >= 1, so 10^p <= 2^k <=> bitlen(10^p) <= k
    int bl = HBig::pow10(p).bitlen();
    return (bl + 1 + 31) / 32;
}

}  // namespace uph
