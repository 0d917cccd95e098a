// devsw.hpp -- development switches: environment integers read ONCE per process
// and cached, so no launch path calls getenv().  Switches select measured alternatives or
// diagnostics; none changes results (the cost-isolation switches that would are compiled in only
// with -DEATSS_DEVTOOLS).
#pragma once
#include <cstdlib>
#include <map>
#include <mutex>
#include <string>

namespace eatss {
inline int devsw(const char *name, int dflt) {
    static std::mutex mu;
    static std::map<std::string, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(name);
    if (it != cache.end()) return it->second;
    const char *e = getenv(name);
    const int v = e ? atoi(e) : dflt;
    cache.emplace(name, v);
    return v;
}
}  // namespace eatss
