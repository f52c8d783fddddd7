// Internal helpers shared by the libmobius translation units.
#pragma once

#include <cstdint>
#include <cstdio>
#include <string>

#include "../../include/mobius.h"

namespace mobius {

void set_error(const char* fmt, ...);

struct Error {
  int code;
};

}  // namespace mobius

#define MOBIUS_FAIL(code, ...)          \
  do {                                  \
    ::mobius::set_error(__VA_ARGS__);   \
    return (code);                      \
  } while (0)

#define MOBIUS_CHECK_ARG(cond, ...)                          \
  do {                                                       \
    if (!(cond)) MOBIUS_FAIL(MOBIUS_EINVAL, __VA_ARGS__);    \
  } while (0)
