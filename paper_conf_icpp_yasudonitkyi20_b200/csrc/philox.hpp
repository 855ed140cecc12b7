// Counter-based RNG for the host GA: Philox4x32 with 10 rounds (Salmon et al.,
// SC'11).  The library's own implementation (the oracle has a separate one;
// both are pinned by the Random123 known-answer vectors in tests/golden).
#pragma once
#include <array>
#include <cstdint>

namespace absb {

struct Philox4x32x10 {
    using Block = std::array<uint32_t, 4>;
    static constexpr uint32_t kMulA = 0xD2511F53u, kMulB = 0xCD9E8D57u;
    static constexpr uint32_t kWeylA = 0x9E3779B9u, kWeylB = 0xBB67AE85u;

    uint32_t k0, k1;
    explicit Philox4x32x10(uint64_t seed) : k0(static_cast<uint32_t>(seed)), k1(static_cast<uint32_t>(seed >> 32)) {}

    Block operator()(Block x) const
    {
        uint32_t a = k0, b = k1;
        for (int round = 0; round < 10; ++round) {
            const uint64_t pa = static_cast<uint64_t>(kMulA) * x[0];
            const uint64_t pb = static_cast<uint64_t>(kMulB) * x[2];
            x = Block{static_cast<uint32_t>(pb >> 32) ^ x[1] ^ a, static_cast<uint32_t>(pb),
                      static_cast<uint32_t>(pa >> 32) ^ x[3] ^ b, static_cast<uint32_t>(pa)};
            a += kWeylA;
            b += kWeylB;
        }
        return x;
    }
};

}  // namespace absb
