// fault.hpp — crash injection for the crash-consistency tests (SURVEY §4 "Integration").
//
// PCC_FAULT=<point>:<n> makes the process SIGKILL itself at the n-th occurrence (1-based) of
// <point>.  SIGKILL keeps the page cache, so this tests the ORDER of the writes (FORMAT.md's
// commit order); torn bytes are injected separately (mid_pointer writes half a record).
//   chunk        after a chunk landed in host memory / the file
//   header       before a COMPLETE slot header is written
//   pointer      before a pointer record is written
//   mid_pointer  after writing the first half of a pointer record
//   k1_fail      (not a crash) the n-th K1 window launch reports a launch failure
#pragma once
#include <csignal>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <unistd.h>

namespace pcc {

inline bool fault_hit(const char *point) {
    static std::mutex mu;
    static bool parsed = false;
    static std::string want;
    static long target = 0, seen = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!parsed) {
        parsed = true;
        if (const char *e = std::getenv("PCC_FAULT")) {
            const char *colon = std::strchr(e, ':');
            if (colon) {
                want.assign(e, colon - e);
                target = std::strtol(colon + 1, nullptr, 10);
            }
        }
    }
    if (want.empty() || want != point) return false;
    return ++seen == target;
}

[[noreturn]] inline void fault_die() {
    ::kill(::getpid(), SIGKILL);
    std::abort();
}

}  // namespace pcc
