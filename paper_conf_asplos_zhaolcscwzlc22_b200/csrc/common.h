// Shared host-side helpers: status codes, thread-local error, checks.
#pragma once
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <stdexcept>
#include <string>

#include "naspipe.h"

namespace naspipe {

// Error carrying a naspipe_status; thrown inside the library, converted at the C ABI.
struct Error : std::runtime_error {
  int code;
  Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

std::string strfmt(const char* fmt, ...);
void set_last_error(const std::string& msg);

#define NP_REQUIRE(cond, code, ...)                                         \
  do {                                                                      \
    if (!(cond)) throw ::naspipe::Error((code), ::naspipe::strfmt(__VA_ARGS__)); \
  } while (0)

}  // namespace naspipe
