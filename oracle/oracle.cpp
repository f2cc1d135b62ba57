/* oracle.cpp — plain, slow, obviously-correct CPU oracle for the SEPO hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. It shares no code, header, table or constant
 * with the CUDA path (paper_conf_ipps_mokhtaris17_b200/), and neither imports the other.
 *
 * What the method computes (PAPER.md = /root/reference/PAPER.md, cited as P:L<line>):
 *   SEPO is exact — postponement only changes when a request is served — so the
 *   result of a SEPO job is the plain group-by of the input multiset:
 *   * combining method (PVC P:L73 "<url,1> inserted n times -> <url,n>"; WC P:L217):
 *       R = { (k, sum_{i: key_i = k} v_i mod 2^64) }      (combiner fixed to u64 wrapping sum,
 *                                                          DESIGN.md reading R1)
 *   * multi-valued method (P:L115-117, P:L133 google.com -> {a.html, c.html, d.html}):
 *       R = { (k, multiset{ v_i : key_i = k }) }
 *   * stream-compaction re-issue (the paper's "iterate over records not yet
 *     processed"): the sub-sequence of records whose postponed bit is 1, in input order.
 *   * sepo_sim_*: the paper's pass loop step by step, single
 *     threaded, with a heap of a fixed byte capacity; used to check the paper's claim that the
 *     multi-pass result equals the group-by and to report the sequential pass count.
 * Canonical output: keys sorted as unsigned-byte strings (std::string order, shorter prefix
 * first); each value list sorted the same way.
 */
#include <stdint.h>
#include <string.h>
#include <algorithm>
#include <string>
#include <unordered_map>
#include <vector>

namespace {
typedef std::unordered_map<std::string, uint64_t> CombineMap;
typedef std::unordered_map<std::string, std::vector<std::string>> GroupMap;

// Value of record i as an unsigned integer: width 0 => 1 (Word Count / PVC);
// width w in 1..8 => w little-endian bytes at vals + w*i (zero-extended).
uint64_t value_u64(const uint8_t* vals, uint32_t w, uint64_t i) {
    if (w == 0) return 1;
    uint64_t v = 0;
    for (uint32_t b = 0; b < w; ++b) v |= (uint64_t)vals[(uint64_t)w * i + b] << (8 * b);
    return v;
}
std::string key_of(const uint8_t* keys, const uint64_t* offs, uint64_t i) {
    return std::string((const char*)keys + offs[i], (size_t)(offs[i + 1] - offs[i]));
}
// Value bytes of record i for the multi-valued method: val_offs given => bytes
// vals[vo[i]..vo[i+1]); else w bytes at vals + w*i.
std::string val_bytes_of(const uint8_t* vals, const uint64_t* vo, uint32_t w, uint64_t i) {
    if (vo) return std::string((const char*)vals + vo[i], (size_t)(vo[i + 1] - vo[i]));
    return std::string((const char*)vals + (uint64_t)w * i, w);
}

struct Combine { CombineMap m; std::vector<std::string> sorted; };
struct Group { GroupMap m; std::vector<std::string> sorted; };
}  // namespace

extern "C" {

/* ------------------------------------------------------------------ combining group-by */
void* oracle_combine_new(void) { return new Combine(); }
void oracle_combine_free(void* h) { delete (Combine*)h; }

/* m[key_i] += v_i for i in [0, n) — P:L75 "its value is combined with the currently stored
   value of the key", "update the value of the existing bucket entry". */
void oracle_combine_add(void* h, const uint8_t* keys, const uint64_t* offs, const uint8_t* vals, uint32_t vw, uint64_t n) {
    Combine* c = (Combine*)h;
    for (uint64_t i = 0; i < n; ++i) c->m[key_of(keys, offs, i)] += value_u64(vals, vw, i);
}
/* number of distinct keys; *key_bytes = total bytes of the distinct keys */
/* Word count on raw text (the paper's WC; reading R20): a word is a maximal run of bytes
 * other than ' ', '\n', '\t', '\r'; each occurrence adds 1 to its word. */
void oracle_combine_add_text(void* h, const uint8_t* text, uint64_t n) {
    CombineMap& m = ((Combine*)h)->m;
    std::string word;
    for (uint64_t i = 0; i <= n; ++i) {
        const bool sep = i == n || text[i] == ' ' || text[i] == '\n' || text[i] == '\t' || text[i] == '\r';
        if (!sep) { word.push_back((char)text[i]); continue; }
        if (!word.empty()) { m[word] += 1; word.clear(); }
    }
}
uint64_t oracle_combine_size(void* h, uint64_t* key_bytes) {
    Combine* c = (Combine*)h;
    c->sorted.clear();
    c->sorted.reserve(c->m.size());
    uint64_t kb = 0;
    for (auto& kv : c->m) { c->sorted.push_back(kv.first); kb += kv.first.size(); }
    std::sort(c->sorted.begin(), c->sorted.end());
    *key_bytes = kb;
    return c->sorted.size();
}
/* canonical result (call oracle_combine_size first): keys CSR + values */
void oracle_combine_result(void* h, uint8_t* keys, uint64_t* offs, uint64_t* vals) {
    Combine* c = (Combine*)h;
    uint64_t o = 0;
    for (size_t i = 0; i < c->sorted.size(); ++i) {
        const std::string& k = c->sorted[i];
        offs[i] = o;
        memcpy(keys + o, k.data(), k.size());
        o += k.size();
        vals[i] = c->m[k];
    }
    offs[c->sorted.size()] = o;
}
/* ------------------------------------------------------------------ multi-valued group-by */
void* oracle_group_new(void) { return new Group(); }
void oracle_group_free(void* h) { delete (Group*)h; }
/* m[key_i].push_back(val_i) — P:L117 "a separate list of values is associated with each key";
   P:L133 one pair per occurrence (duplicates kept: DESIGN.md reading R4). */
void oracle_group_add(void* h, const uint8_t* keys, const uint64_t* offs, const uint8_t* vals, const uint64_t* val_offs,
                      uint32_t vw, uint64_t n) {
    Group* g = (Group*)h;
    for (uint64_t i = 0; i < n; ++i) g->m[key_of(keys, offs, i)].push_back(val_bytes_of(vals, val_offs, vw, i));
}
/* returns #keys; *key_bytes, *n_vals, *val_bytes totals. Sorts keys and each list. */
uint64_t oracle_group_size(void* h, uint64_t* key_bytes, uint64_t* n_vals, uint64_t* val_bytes) {
    Group* g = (Group*)h;
    g->sorted.clear();
    uint64_t kb = 0, nv = 0, vb = 0;
    for (auto& kv : g->m) {
        g->sorted.push_back(kv.first);
        kb += kv.first.size();
        std::sort(kv.second.begin(), kv.second.end());
        nv += kv.second.size();
        for (auto& v : kv.second) vb += v.size();
    }
    std::sort(g->sorted.begin(), g->sorted.end());
    *key_bytes = kb; *n_vals = nv; *val_bytes = vb;
    return g->sorted.size();
}
/* keys CSR, list_offs[n_keys+1] (into the value sequence), values CSR (val_offs[n_vals+1]) */
void oracle_group_result(void* h, uint8_t* keys, uint64_t* offs, uint64_t* list_offs, uint8_t* vals, uint64_t* val_offs) {
    Group* g = (Group*)h;
    uint64_t ko = 0, li = 0, vo = 0;
    for (size_t i = 0; i < g->sorted.size(); ++i) {
        const std::string& k = g->sorted[i];
        offs[i] = ko; memcpy(keys + ko, k.data(), k.size()); ko += k.size();
        list_offs[i] = li;
        for (auto& v : g->m[k]) { val_offs[li] = vo; memcpy(vals + vo, v.data(), v.size()); vo += v.size(); ++li; }
    }
    offs[g->sorted.size()] = ko;
    list_offs[g->sorted.size()] = li;
    val_offs[li] = vo;
}

/* ------------------------------------------------------------------ compaction (a9)
 * The re-issue set of a pass: records i with bit (i & 31) of bitmap[i >> 5] == 1 (postponed,
 * SURVEY §8(b) bitmap convention), in input order, with key/value offsets rebased to 0.
 * val_offs == NULL => fixed width vw (vw == 0: no values). Returns the number gathered. */
uint64_t oracle_compact(const uint8_t* keys, const uint64_t* offs, const uint8_t* vals, const uint64_t* val_offs, uint32_t vw,
                        uint64_t n, const uint32_t* bitmap, uint8_t* out_keys, uint64_t* out_offs, uint8_t* out_vals,
                        uint64_t* out_val_offs) {
    uint64_t m = 0, ko = 0, vo = 0;
    for (uint64_t i = 0; i < n; ++i) {
        if (!((bitmap[i >> 5] >> (i & 31)) & 1u)) continue;
        uint64_t kl = offs[i + 1] - offs[i];
        out_offs[m] = ko; memcpy(out_keys + ko, keys + offs[i], kl); ko += kl;
        if (val_offs) {
            uint64_t vl = val_offs[i + 1] - val_offs[i];
            out_val_offs[m] = vo; memcpy(out_vals + vo, vals + val_offs[i], vl); vo += vl;
        } else if (vw) {
            memcpy(out_vals + (uint64_t)vw * m, vals + (uint64_t)vw * i, vw);
        }
        ++m;
    }
    out_offs[m] = ko;
    if (val_offs) out_val_offs[m] = vo;
    return m;
}

/* ------------------------------------------------------------------ SEPO, sequential
 * The paper's combining pass loop, one request at a time:
 *   for each pass: for each record not yet processed, in input order:
 *     key resident in this pass's heap  -> combine value, SUCCESS (bit set)
 *     else allocate entry_bytes(key)    -> if it fits: insert <k,v>, SUCCESS
 *                                          else POSTPONE (record stays unprocessed)
 *   end of pass: copy every resident pair to CPU memory, free the heap
 * Entries are allocated "exactly as large as they need to be": entry_bytes = overhead +
 * key length. heap_bytes is the heap capacity. Returns the pass count (or -1 if one record can
 * never fit); postponed[p] = records postponed in pass p (up to max_passes). The final result
 * (generations concatenated) goes into `out` (an oracle_combine handle); *dup_keys counts keys
 * seen in more than one generation (the paper's guarantee P:L77/P:L79 says 0). */
int64_t oracle_sepo_sim_combine(const uint8_t* keys, const uint64_t* offs, const uint8_t* vals, uint32_t vw, uint64_t n,
                                uint64_t heap_bytes, uint64_t overhead, uint64_t* postponed, uint64_t max_passes,
                                void* out, uint64_t* dup_keys) {
    std::vector<uint8_t> processed(n, 0);  // the paper's bitmap, 1 bit per input record
    CombineMap cpu;                          // pairs copied back to CPU memory
    uint64_t remaining = n, pass = 0, dups = 0;
    while (remaining > 0) {
        CombineMap heap; uint64_t used = 0, post = 0;
        for (uint64_t i = 0; i < n; ++i) {
            if (processed[i]) continue;
            std::string k = key_of(keys, offs, i);
            auto it = heap.find(k);
            if (it != heap.end()) { it->second += value_u64(vals, vw, i); processed[i] = 1; continue; }
            uint64_t sz = overhead + k.size();
            if (sz > heap_bytes) return -1;
            if (used + sz <= heap_bytes) { used += sz; heap.emplace(k, value_u64(vals, vw, i)); processed[i] = 1; }
            else ++post;
        }
        if (pass < max_passes) postponed[pass] = post;
        ++pass;
        for (auto& kv : heap) {  // copy the heap back to CPU memory and free it
            auto r = cpu.emplace(kv.first, kv.second);
            if (!r.second) { ++dups; r.first->second += kv.second; }
        }
        remaining = post;
    }
    Combine* o = (Combine*)out;
    for (auto& kv : cpu) o->m[kv.first] += kv.second;
    *dup_keys = dups;
    return (int64_t)pass;
}

/* The multi-valued pass loop, one request at a time. Keys and values live in
 * separate storage: a key entry costs key_overhead + klen bytes, a value costs
 * val_overhead + vlen bytes, both from one heap of heap_bytes. A value whose key is resident is
 * appended if its bytes fit, else POSTPONE; a new key needs key + value bytes. At the end of a
 * pass, all values and every key with no pending (postponed) value are copied to CPU memory and
 * freed; keys with pending values stay resident. If a pass makes no progress
 * (retained keys starve the heap — the paper is silent, reading R14) every key is
 * evicted and may reappear in a later generation; the lists are then concatenated. */
int64_t oracle_sepo_sim_group(const uint8_t* keys, const uint64_t* offs, const uint8_t* vals, const uint64_t* val_offs,
                              uint32_t vw, uint64_t n, uint64_t heap_bytes, uint64_t key_overhead, uint64_t val_overhead,
                              uint64_t* postponed, uint64_t max_passes, void* out, uint64_t* forced_full) {
    std::vector<uint8_t> processed(n, 0);
    GroupMap cpu;
    std::unordered_map<std::string, uint64_t> resident_keys;  // key -> bytes of its key entry
    uint64_t remaining = n, pass = 0, forced = 0, key_used = 0;
    while (remaining > 0) {
        GroupMap heap_vals;  // values inserted this pass (value storage is fully evicted each pass)
        for (auto& kv : resident_keys) heap_vals[kv.first];
        uint64_t used = key_used, post = 0;
        std::unordered_map<std::string, int> pending;
        for (uint64_t i = 0; i < n; ++i) {
            if (processed[i]) continue;
            std::string k = key_of(keys, offs, i);
            std::string v = val_bytes_of(vals, val_offs, vw, i);
            uint64_t vsz = val_overhead + v.size();
            if (resident_keys.count(k)) {
                if (used + vsz <= heap_bytes) { used += vsz; heap_vals[k].push_back(v); processed[i] = 1; }
                else { ++post; pending[k] = 1; }
                continue;
            }
            uint64_t ksz = key_overhead + k.size();
            if (ksz + vsz > heap_bytes) return -1;
            if (used + ksz + vsz <= heap_bytes) {
                used += ksz + vsz; key_used += ksz; resident_keys[k] = ksz;
                heap_vals[k].push_back(v); processed[i] = 1;
            } else ++post;
        }
        if (pass < max_passes) postponed[pass] = post;
        ++pass;
        bool progress = post < remaining;
        for (auto& kv : heap_vals) {  // all value pages go to CPU memory (P:L165 (i))
            auto& dst = cpu[kv.first];
            dst.insert(dst.end(), kv.second.begin(), kv.second.end());
        }
        // keys with no pending values are evicted; pending keys stay resident
        std::unordered_map<std::string, uint64_t> keep;
        if (progress)
            for (auto& kv : resident_keys) if (pending.count(kv.first)) keep.insert(kv);
        if (!progress) ++forced;
        resident_keys.swap(keep);
        key_used = 0;
        for (auto& kv : resident_keys) key_used += kv.second;
        remaining = post;
    }
    Group* o = (Group*)out;
    for (auto& kv : cpu) { auto& d = o->m[kv.first]; d.insert(d.end(), kv.second.begin(), kv.second.end()); }
    *forced_full = forced;
    return (int64_t)pass;
}

}  // extern "C"
