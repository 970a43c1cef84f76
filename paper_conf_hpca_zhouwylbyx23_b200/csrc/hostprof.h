// Host-time breakdown of the swap calls, compiled in only for an experimental
// build (MPRESS_NVCC_FLAGS=-DMPRESS_HOSTPROF, tools/hostcost.py --breakdown);
// the product build has empty macros.  Sections accumulate nanoseconds per
// call site and print to stderr at process exit.
#pragma once

#ifdef MPRESS_HOSTPROF
#include <chrono>
#include <cstdint>
#include <cstdio>

namespace mpress {
struct HostProf {
  static constexpr int kN = 16;
  const char* name[kN] = {};
  uint64_t ns[kN] = {};
  uint64_t n[kN] = {};
  ~HostProf() {
    for (int i = 0; i < kN; ++i)
      if (n[i]) fprintf(stderr, "[hostprof] %-28s %8.3f us/call (%llu calls)\n", name[i], ns[i] / 1e3 / n[i],
                        (unsigned long long)n[i]);
  }
};
inline HostProf& hostprof() {
  static HostProf p;
  return p;
}
inline uint64_t hp_now() {
  return std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch()).count();
}
}  // namespace mpress
#define HP_START() uint64_t _hp_t = mpress::hp_now()
#define HP_LAP(i, label)                                  \
  do {                                                    \
    const uint64_t _hp_n = mpress::hp_now();              \
    auto& _p = mpress::hostprof();                        \
    _p.name[i] = label;                                   \
    _p.ns[i] += _hp_n - _hp_t;                            \
    ++_p.n[i];                                            \
    _hp_t = _hp_n;                                        \
  } while (0)
#else
#define HP_START() \
  do {             \
  } while (0)
#define HP_LAP(i, label) \
  do {                   \
  } while (0)
#endif
