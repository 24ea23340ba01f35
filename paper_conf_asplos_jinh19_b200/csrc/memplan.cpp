// memplan.cpp -- HMMS static memory planning (§4.4), the library's own
// implementation (it shares nothing with oracle/memplan.py).
//
// "The static memory planning algorithm steps through the list of operations in the serialized
//  computation graph to allocate memory space to each tensor storage object (TSO). It uses first-fit
//  memory allocation ... Memory is allocated to TSO only for the minimum duration required".
//
// Input: per TSO its byte size and the serialized op indices of its first (allocation) and last
// (release) use.  Walking the ops in order, at op t every TSO whose last use is < t is released
// first (its bytes rejoin the free list, coalesced with free neighbours), then every TSO first used
// at t is placed, in TSO index order, at the LOWEST offset of a free hole it fits in (first fit);
// the pool grows at its end when no hole fits.  Output: offsets and the pool size (high-water mark).
#include <algorithm>
#include <cstdint>
#include <map>
#include <vector>

#include "internal.h"

using namespace splitcnn;

extern "C" splitcnn_status_t splitcnn_memplan(int32_t n, const int64_t *bytes, const int32_t *first_use,
                                              const int32_t *last_use, int64_t align, int64_t *offsets,
                                              int64_t *pool_bytes) {
    if (n < 0 || (n > 0 && (!bytes || !first_use || !last_use || !offsets)) || !pool_bytes)
        return fail(SPLITCNN_ERR_INVALID_VALUE, "memplan: null argument");
    if (align <= 0 || (align & (align - 1))) return fail(SPLITCNN_ERR_INVALID_VALUE, "memplan: align must be a power of 2");
    int32_t T = 0;
    for (int i = 0; i < n; ++i) {
        if (bytes[i] < 0 || first_use[i] < 0 || last_use[i] < first_use[i])
            return fail(SPLITCNN_ERR_INVALID_VALUE, "memplan: bad TSO (negative size or last_use < first_use)");
        T = std::max(T, last_use[i] + 1);
    }
    std::vector<std::vector<int>> born(T), dies(T);
    for (int i = 0; i < n; ++i) {
        born[first_use[i]].push_back(i);
        dies[last_use[i]].push_back(i);
    }
    std::map<int64_t, int64_t> holes;   // offset -> size, disjoint, coalesced, all below `top`
    int64_t top = 0, peak = 0;
    auto size_of = [&](int i) { return (bytes[i] + align - 1) / align * align; };
    auto release = [&](int i) {
        int64_t off = offsets[i], sz = size_of(i);
        if (sz == 0) return;
        auto nx = holes.lower_bound(off);
        if (nx != holes.end() && off + sz == nx->first) {   // merge with the following hole
            sz += nx->second;
            nx = holes.erase(nx);
        }
        if (nx != holes.begin()) {                           // merge with the preceding hole
            auto pv = std::prev(nx);
            if (pv->first + pv->second == off) {
                off = pv->first;
                sz += pv->second;
                holes.erase(pv);
            }
        }
        if (off + sz == top) top = off;                      // the free tail shrinks the live top
        else holes[off] = sz;
        while (!holes.empty()) {                             // a hole now touching the top is absorbed
            auto last = std::prev(holes.end());
            if (last->first + last->second != top) break;
            top = last->first;
            holes.erase(last);
        }
    };
    for (int32_t t = 0; t < T; ++t) {
        if (t > 0)
            for (int i : dies[t - 1]) release(i);           // last use < t
        for (int i : born[t]) {
            const int64_t sz = size_of(i);
            if (sz == 0) { offsets[i] = 0; continue; }
            auto it = holes.begin();
            for (; it != holes.end(); ++it)
                if (it->second >= sz) break;
            if (it != holes.end()) {
                offsets[i] = it->first;
                const int64_t rest = it->second - sz, roff = it->first + sz;
                holes.erase(it);
                if (rest > 0) holes[roff] = rest;
            } else {
                offsets[i] = top;
                top += sz;
            }
            peak = std::max(peak, top);
        }
    }
    *pool_bytes = peak;
    return SPLITCNN_OK;
}
