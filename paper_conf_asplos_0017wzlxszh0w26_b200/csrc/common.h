// Shared host-side helpers of libbat: status/error plumbing and small utilities.
#pragma once

#include <cstdint>
#include <cstdio>
#include <cstring>
#include <stdexcept>
#include <string>

#include "bat.h"

namespace bat {

// Thread-local last-error message (bat_last_error).
void set_error(const std::string& msg);
const char* last_error();

// Internal exception carrying a bat_status; caught at the ABI boundary.
struct Error : std::runtime_error {
  bat_status status;
  Error(bat_status s, const std::string& m) : std::runtime_error(m), status(s) {}
};

[[noreturn]] inline void fail(bat_status s, const std::string& m) { throw Error(s, m); }

#define BAT_REQUIRE(cond, msg)                                                       \
  do {                                                                               \
    if (!(cond)) ::bat::fail(BAT_E_INVAL, std::string("invalid argument: ") + (msg)); \
  } while (0)

// Map any exception to a status and record the message.
template <class F>
bat_status guarded(F&& f) {
  try {
    f();
    return BAT_OK;
  } catch (const Error& e) {
    set_error(e.what());
    return e.status;
  } catch (const std::bad_alloc&) {
    set_error("host allocation failed");
    return BAT_E_OOM;
  } catch (const std::exception& e) {
    set_error(e.what());
    return BAT_E_INVAL;
  }
}

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

constexpr int kPageTokens = 16;
constexpr int kKtilePages = 8;
constexpr int kKtile = kPageTokens * kKtilePages;  // 128 key slots per k-tile
constexpr int kQtileRows = 128;                    // packed q-tile rows (tokens x group)
constexpr int32_t kInvalidOrd = 0x7fffffff;
constexpr int32_t kZeroPage = INT32_MIN;           // page-list padding -> the all-zero page

enum Seg : int32_t { SEG_USER = -1, SEG_INSTR = -2, SEG_HEADER = -3 };

// head_dim padded to the tensor-core operand width (64-element, 128-byte swizzle rows)
inline int head_dim_pad(int d) { return d <= 64 ? 64 : 128; }

}  // namespace bat
