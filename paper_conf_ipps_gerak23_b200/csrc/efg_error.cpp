// efg_error.cpp — thread-local error message for the C ABI (efg_last_error).
#include <string>

#include "efg_internal.h"

namespace {
thread_local std::string g_last_error;
}

namespace efg {
efg_status set_error(efg_status s, const std::string &msg)
{
    g_last_error = msg;
    return s;
}
void clear_error() { g_last_error.clear(); }
}  // namespace efg

extern "C" const char *efg_last_error(void) { return g_last_error.c_str(); }
extern "C" const char *efg_version(void) { return "efg-b200 0.1 (sm_100a)"; }
