// gmbe_api.cu -- error plumbing of the C ABI (gmbe_last_error) and ABI version query.
#include <string>

#include "gmbe_internal.cuh"

namespace {
thread_local std::string g_last_error;
}

int gmbe_set_error(int code, const std::string& msg) {
  g_last_error = msg;
  return code;
}

extern "C" const char* gmbe_last_error(void) { return g_last_error.c_str(); }
