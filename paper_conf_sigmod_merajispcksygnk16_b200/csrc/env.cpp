// BLU_* tuning / test knobs read once per API call. Every public entry point calls env_snapshot(),
// which copies this thread's view of the BLU_* environment variables (one pass over environ, and
// only when environ changed since the last snapshot); benv() then answers from the copy, so the
// per-launch paths do not scan the environment a dozen times per execute (C1: ~10 getenv per call).
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <string>
#include <utility>
#include <vector>

#include "blu_internal.h"

extern char** environ;

namespace blu {

namespace {
struct Snap {
  bool valid = false;
  uint64_t fp = 0;
  std::vector<std::pair<std::string, std::string>> kv;
};
thread_local Snap t_snap;

// setenv/putenv/unsetenv replace an entry pointer, change the count or reallocate the array
uint64_t environ_fingerprint() {
  uint64_t f = (uint64_t)(uintptr_t)environ, n = 0;
  for (char** e = environ; e && *e; ++e, ++n) f = (f ^ (uint64_t)(uintptr_t)*e) * 1099511628211ull;
  return f ^ (n << 52);
}
}  // namespace

void env_snapshot() {
  const uint64_t f = environ_fingerprint();
  if (t_snap.valid && f == t_snap.fp) return;
  t_snap.kv.clear();
  for (char** e = environ; e && *e; ++e) {
    const char* s = *e;
    if (strncmp(s, "BLU_", 4) != 0) continue;
    const char* eq = strchr(s, '=');
    if (!eq) continue;
    t_snap.kv.emplace_back(std::string(s, eq - s), std::string(eq + 1));
  }
  t_snap.fp = f;
  t_snap.valid = true;
}

const char* benv(const char* name) {
  if (!t_snap.valid) env_snapshot();
  for (const auto& kv : t_snap.kv)
    if (kv.first == name) return kv.second.c_str();
  return nullptr;
}

}  // namespace blu
