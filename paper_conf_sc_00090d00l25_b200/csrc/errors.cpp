// Thread-local last-error message of the C ABI (include/gllm.h).
#include <cstdarg>
#include <cstdio>
#include <string>

#include "common.h"

namespace {
thread_local std::string g_last_error;
}

namespace gllm {
int set_error(int code, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  std::vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}
}  // namespace gllm

extern "C" const char* gllm_last_error(void) { return g_last_error.c_str(); }
extern "C" const char* gllm_version(void) { return "gllm-b200 0.1 sm_100a"; }
