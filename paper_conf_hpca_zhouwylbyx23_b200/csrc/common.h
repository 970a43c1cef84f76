// Internal helpers shared by the libmpress translation units (not part of the ABI).
#pragma once

#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <string>

#include "../../include/mpress.h"

namespace mpress {

// Thread-local message behind mpress_last_error().
void set_error(const char* fmt, ...) __attribute__((format(printf, 1, 2)));
int fail(int code, const char* fmt, ...) __attribute__((format(printf, 2, 3)));

inline uint64_t roundup(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

// Checked a+b on uint64 (returns false on overflow).
inline bool add_ok(uint64_t a, uint64_t b, uint64_t* r) {
  return !__builtin_add_overflow(a, b, r);
}

}  // namespace mpress

#define MP_TRY(expr)                   \
  do {                                 \
    int _rc = (expr);                  \
    if (_rc != MPRESS_OK) return _rc;  \
  } while (0)
