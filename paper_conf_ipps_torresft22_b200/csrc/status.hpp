// status.hpp -- thread-local last-error plumbing shared by the C-ABI entry points.
#pragma once
#include <cstdarg>
#include <cstdio>
#include <string>

#include "spread.h"

namespace paper {

void set_last_error(const char* fmt, ...) __attribute__((format(printf, 1, 2)));
void clear_last_error();

// Return `st` after recording a formatted message.
#define PAPER_FAIL(st, ...)                   \
    do {                                      \
        ::paper::set_last_error(__VA_ARGS__); \
        return (st);                          \
    } while (0)

}  // namespace paper
