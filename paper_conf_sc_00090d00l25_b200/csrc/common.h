// Internal helpers shared by the library's translation units (not part of the ABI).
#pragma once
#include <cstdarg>
#include <cstdio>
#include <string>

#include "gllm.h"

namespace gllm {

int set_error(int code, const char* fmt, ...);

}  // namespace gllm

#define GLLM_TRY_BEGIN try {
#define GLLM_TRY_END                                                       \
  }                                                                        \
  catch (const std::bad_alloc&) {                                          \
    return gllm::set_error(GLLM_ENOMEM, "host allocation failed");         \
  }                                                                        \
  catch (const std::exception& e) {                                        \
    return gllm::set_error(GLLM_EINVAL, "exception: %s", e.what());        \
  }                                                                        \
  catch (...) {                                                            \
    return gllm::set_error(GLLM_EINVAL, "unknown exception");              \
  }
