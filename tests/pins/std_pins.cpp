// Independent pins for the oracle: the C++ standard library's own in-place
// algorithms (std::remove, std::copy_if, std::unique).  Compiled by the test
// suite (g++) into a throwaway .so; it shares no code with oracle/ or libds.
//
// compact == std::remove (bitwise ==), select == std::copy_if
// into a fresh vector copied back, unique == std::unique (bitwise ==).
#include <algorithm>
#include <cstddef>
#include <cstdint>
#include <cstring>
#include <vector>

extern "C" {

size_t std_remove(uint32_t* a, size_t n, uint32_t v) {
    return static_cast<size_t>(std::remove(a, a + n, v) - a);
}

size_t std_unique(uint32_t* a, size_t n) {
    return static_cast<size_t>(std::unique(a, a + n) - a);
}

// Keeps words whose bit `keep_bits[i]` is set, via std::copy_if on indices.
size_t std_copy_if_mask(uint32_t* a, size_t n, const uint8_t* keep) {
    std::vector<uint32_t> out;
    std::vector<size_t> idx(n);
    for (size_t i = 0; i < n; ++i) idx[i] = i;
    std::vector<size_t> kept;
    std::copy_if(idx.begin(), idx.end(), std::back_inserter(kept),
                 [&](size_t i) { return keep[i] != 0; });
    for (size_t i : kept) out.push_back(a[i]);
    if (!out.empty()) std::memcpy(a, out.data(), out.size() * sizeof(uint32_t));
    return out.size();
}

}  // extern "C"
