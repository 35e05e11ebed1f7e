// gmbe_api.cu -- error plumbing of the C ABI (gmbe_last_error) and ABI version query.
#include <string>

#include "gmbe_internal.cuh"

#include <atomic>

namespace {
thread_local std::string g_last_error;
std::atomic<unsigned long long> g_launches{0};
}  // namespace

void gmbe_note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

extern "C" uint64_t gmbe_kernel_launch_count(void) { return g_launches.load(); }

int gmbe_set_error(int code, const std::string& msg) {
  g_last_error = msg;
  return code;
}

extern "C" const char* gmbe_last_error(void) { return g_last_error.c_str(); }
