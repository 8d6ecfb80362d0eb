// errors.cu — thread-local error message, version string, host-logic self-tests.
#include <cstdarg>
#include <cstdio>
#include <string>

#include "common.cuh"

namespace olap {

static thread_local std::string g_err;

int set_error(int status, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_err = buf;
    return status;
}

void clear_error() { g_err.clear(); }

}  // namespace olap

extern "C" {

const char* olap_last_error(void) { return olap::g_err.c_str(); }

const char* olap_version(void) { return "paper_conf_ipps_malikrse12_b200 0.1 (sm_100a)"; }

// Not in olap.h: host-only self-test hooks used by tests/test_host_logic.py.
// q[i] = n[i] / d via the FastDiv used on the device.
int olap_selftest_fastdiv(uint32_t d, const uint32_t* n, int64_t count, uint32_t* q) {
    if (d == 0 || !n || !q) return OLAP_E_INVALID;
    olap::FastDiv f = olap::make_fastdiv(d);
    for (int64_t i = 0; i < count; ++i) q[i] = olap::fdiv(n[i], f);
    return OLAP_OK;
}

// The dictionary hash of one key (host implementation; the device one is tested by parity).
uint64_t olap_selftest_hash(const char* bytes, int64_t len) {
    return olap::hash_bytes_host(reinterpret_cast<const unsigned char*>(bytes), len);
}

}  // extern "C"
