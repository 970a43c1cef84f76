// Error reporting and version for the C ABI (include/mpress.h "Conventions").
#include <cstdarg>
#include <cstdio>
#include <string>

#include "common.h"

namespace mpress {

static thread_local std::string g_last_error;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
}

int fail(int code, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}

}  // namespace mpress

extern "C" const char* mpress_last_error(void) { return mpress::g_last_error.c_str(); }
extern "C" int mpress_version(void) { return MPRESS_VERSION; }
