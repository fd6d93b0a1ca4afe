// regex.cpp -- regular-expression DPI patterns compiled to one DFA (SURVEY 8(f)
// NEXT-4; PAPER.md P:L132 [SIII.A.2] "For the regular expression we use a
// Deterministic Finite Automata (DFA) implementation"; R#33).
//
// Syntax: literal bytes, escapes \xHH and \<punct>, '.', classes [..] with ranges
// and '^' negation, groups (..), alternation '|', quantifiers '?', '*', '+', {m},
// {m,n} (n <= 64) and {m,} (m <= 64).  Search is unanchored: an occurrence of regex j
// ends at byte x iff some non-empty substring ending at x is in L(j).  A set whose
// longest match is at most 1 024 bytes is walked per packet with a maxlen - 1
// re-walk of the flow's preceding bytes; a longer or unbounded one (maxlen =
// 0xFFFFFFFF) flow-serially from the carried state (dpi_stream.cu k_walk_serial).
//
// Thompson NFA per regex, one shared start state; subset construction over the
// 256 byte values with the start state added to every subset (unanchored); the
// result is written in the DpiHost layout the stream kernels walk (identity byte
// classes, accept flag on the transition entry, CSR output sets).
#include <algorithm>
#include <array>
#include <cstring>
#include <map>
#include <new>
#include <stdexcept>
#include <string>
#include <vector>

#include "nfc_internal.h"

namespace nfc {
namespace {

// The NFA size while repeats are expanded (nested {m,n} multiply) is bounded (beyond:
// NFC_EUNSUP).  Longest-match lengths saturate at REGEX_INF ('*', '+', {m,}); a set whose
// longest match exceeds REGEX_PAR_MAXLEN is walked flow-serially (DpiHost::maxlen =
// 0xFFFFFFFF), the bounded re-walk of the per-packet walk being too long or unbounded.
constexpr long long REGEX_INF = 1LL << 40;
constexpr long long REGEX_PAR_MAXLEN = 1024;
constexpr size_t REGEX_NFA_MAX = 1u << 16;   // NFA states (subset construction cost grows with it)
inline long long sat(long long x) { return x > REGEX_INF ? REGEX_INF : x; }

struct Nfa {
    struct St { std::array<uint64_t, 4> set{}; int out = -1; std::vector<int> eps; int accept = -1; };
    std::vector<St> st;
    int add() { st.emplace_back(); return (int)st.size() - 1; }
};

struct Frag { int in, out; };

struct Parser {
    const uint8_t *p, *e;
    Nfa &n;
    std::string err;
    int maxlen_cur = 0;
    Parser(const uint8_t *b, const uint8_t *end, Nfa &nfa) : p(b), e(end), n(nfa) {}

    static int hexv(uint8_t c) { return c >= '0' && c <= '9' ? c - '0' : c >= 'a' && c <= 'f' ? c - 'a' + 10 : c >= 'A' && c <= 'F' ? c - 'A' + 10 : -1; }
    bool esc(uint8_t &out) {   // after '\'
        if (p >= e) { err = "regex: trailing backslash"; return false; }
        uint8_t c = *p++;
        if (c == 'x') {
            if (e - p < 2 || hexv(p[0]) < 0 || hexv(p[1]) < 0) { err = "regex: bad \\x escape"; return false; }
            out = (uint8_t)(hexv(p[0]) * 16 + hexv(p[1]));
            p += 2;
            return true;
        }
        if ((c >= '0' && c <= '9') || (c >= 'a' && c <= 'z') || (c >= 'A' && c <= 'Z')) { err = "regex: unsupported escape"; return false; }
        out = c;
        return true;
    }
    Frag atom_set(const std::array<uint64_t, 4> &set) {
        int a = n.add(), b = n.add();
        n.st[a].set = set;
        n.st[a].out = b;
        return {a, b};
    }
    // returns fragment and its (min unused) max length in *len
    bool atom(Frag &f, long long &len) {
        uint8_t c = *p++;
        std::array<uint64_t, 4> set{};
        auto put = [&](int b) { set[b >> 6] |= 1ull << (b & 63); };
        if (c == '(') {
            if (!alt(f, len)) return false;
            if (p >= e || *p != ')') { err = "regex: missing ')'"; return false; }
            p++;
            return true;
        }
        if (c == '*' || c == '+') { err = "regex: misplaced quantifier"; return false; }
        if (c == '^' || c == '$') { err = "regex: anchors ('^', '$' outside a class) not supported"; return false; }
        if (c == ')' || c == '?' || c == '{' || c == '|') { err = "regex: misplaced metacharacter"; return false; }
        if (c == '.') { for (int b = 0; b < 256; b++) put(b); }
        else if (c == '\\') { uint8_t x; if (!esc(x)) return false; put(x); }
        else if (c == '[') {
            bool neg = p < e && *p == '^';
            if (neg) p++;
            bool first = true;
            while (p < e && (*p != ']' || first)) {
                first = false;
                uint8_t lo = *p++;
                if (lo == '\\' && !esc(lo)) return false;
                uint8_t hi = lo;
                if (p + 1 < e && *p == '-' && p[1] != ']') {
                    p++;
                    hi = *p++;
                    if (hi == '\\' && !esc(hi)) return false;
                    if (hi < lo) { err = "regex: bad class range"; return false; }
                }
                for (int b = lo; b <= hi; b++) put(b);
            }
            if (p >= e) { err = "regex: missing ']'"; return false; }
            p++;
            if (neg) for (auto &w : set) w = ~w;
        } else put(c);
        f = atom_set(set);
        len = 1;
        return true;
    }
    bool number(int &v) {
        if (p >= e || *p < '0' || *p > '9') return false;
        v = 0;
        while (p < e && *p >= '0' && *p <= '9') { v = v * 10 + (*p++ - '0'); if (v > 1000) return false; }
        return true;
    }
    // copy of a sub-NFA (states [lo, hi) with entry in, exit out)
    Frag clone(int lo, int hi, Frag f) {
        int base = (int)n.st.size();
        for (int s = lo; s < hi; s++) {
            Nfa::St c = n.st[s];
            if (c.out >= 0) c.out += base - lo;
            for (int &x : c.eps) x += base - lo;
            n.st.push_back(c);
        }
        return {f.in + base - lo, f.out + base - lo};
    }
    bool piece(Frag &f, long long &len) {
        int lo = (int)n.st.size();
        if (!atom(f, len)) return false;
        int hi = (int)n.st.size();
        while (p < e && (*p == '?' || *p == '{' || *p == '*' || *p == '+')) {
            int m = 0, M = 0;
            bool unb = false;                        // '*', '+', {m,}: no upper bound
            if (*p == '?') { p++; m = 0; M = 1; }
            else if (*p == '*') { p++; m = 0; unb = true; }
            else if (*p == '+') { p++; m = 1; unb = true; }
            else {
                p++;
                if (!number(m)) { err = "regex: bad {m,n}"; return false; }
                M = m;
                if (p < e && *p == ',') {
                    p++;
                    if (p < e && *p == '}') unb = true;
                    else if (!number(M)) { err = "regex: bad {m,n}"; return false; }
                }
                if (p >= e || *p != '}' || m > 64 || (!unb && (M < m || M > 64 || M == 0))) {
                    err = "regex: bad {m,n} (need 0 <= m <= n <= 64, n > 0; {m,} with m <= 64)";
                    return false;
                }
                p++;
            }
            const int copies = unb ? m + 1 : M;      // unbounded: m mandatory copies + one looped
            if (n.st.size() + (size_t)(hi - lo) * (size_t)copies + 2 * (size_t)copies + 4 > REGEX_NFA_MAX) {
                err = "regex: NFA above 2^16 states not supported";
                return false;
            }
            // expand: every copy is cloned from the untouched fragment before any is wired
            std::vector<Frag> cp{f};
            for (int k = 1; k < copies; k++) cp.push_back(clone(lo, hi, f));
            const long long olen = len;
            int s0 = n.add(), cur = s0;
            if (unb) {
                for (int k = 0; k < m; k++) {            // the mandatory copies
                    n.st[cur].eps.push_back(cp[k].in);
                    int nx = n.add();
                    n.st[cp[k].out].eps.push_back(nx);
                    cur = nx;
                }
                const int ex = n.add();                  // the loop: zero or more further copies
                n.st[cur].eps.push_back(cp[m].in);
                n.st[cur].eps.push_back(ex);
                n.st[cp[m].out].eps.push_back(cur);
                f = {s0, ex};
                len = REGEX_INF;
            } else {
                std::vector<int> skips;
                for (int k = 0; k < M; k++) {
                    n.st[cur].eps.push_back(cp[k].in);
                    if (k >= m) skips.push_back(cur);
                    int nx = n.add();
                    n.st[cp[k].out].eps.push_back(nx);
                    cur = nx;
                }
                for (int x : skips) n.st[x].eps.push_back(cur);
                f = {s0, cur};
                len = sat(olen * M);
            }
            hi = (int)n.st.size();
        }
        return true;
    }
    bool concat(Frag &f, long long &len) {
        int s = n.add();
        f = {s, s};
        len = 0;
        while (p < e && *p != '|' && *p != ')') {
            Frag g;
            long long l;
            if (!piece(g, l)) return false;
            n.st[f.out].eps.push_back(g.in);
            f.out = g.out;
            len = sat(len + l);
        }
        return true;
    }
    bool alt(Frag &f, long long &len) {
        int s = n.add(), t = n.add();
        f = {s, t};
        len = 0;
        for (;;) {
            Frag g;
            long long l;
            if (!concat(g, l)) return false;
            n.st[s].eps.push_back(g.in);
            n.st[g.out].eps.push_back(t);
            len = std::max(len, l);
            if (p < e && *p == '|') { p++; continue; }
            return true;
        }
    }
};

}  // namespace

static std::string build_regex_dfa_impl(const nfc_dpi_spec &s, DpiHost &o, uint32_t max_states);

// NFC_EUNSUP for messages containing "not supported", NFC_ENOMEM for "out of host memory"
std::string build_regex_dfa(const nfc_dpi_spec &s, DpiHost &o, uint32_t max_states)
{
    try {
        return build_regex_dfa_impl(s, o, max_states);
    } catch (const std::bad_alloc &) {
        return "regex: out of host memory";
    } catch (const std::length_error &) {
        return "regex: out of host memory";
    }
}

static std::string build_regex_dfa_impl(const nfc_dpi_spec &s, DpiHost &o, uint32_t max_states)
{
    if (s.n_patterns == 0 || s.n_patterns > 65535) return "regex: n_patterns must be 1..65535";
    if (!s.blob || !s.off || !s.action) return "regex: NULL pointer";
    Nfa n;
    int start = n.add();
    o.maxlen = 0;
    for (uint32_t j = 0; j < s.n_patterns; j++) {
        if (s.off[j + 1] <= s.off[j]) return "regex: empty expression";
        if (s.action[j] > 1) return "regex: action must be 0 or 1";
        Parser ps(s.blob + s.off[j], s.blob + s.off[j + 1], n);
        Frag f;
        long long len;
        if (!ps.alt(f, len)) return ps.err + " (expression " + std::to_string(j) + ")";
        if (ps.p != ps.e) return "regex: unbalanced ')' (expression " + std::to_string(j) + ")";
        int acc = n.add();
        {   // the language must not contain the empty string (an occurrence is >= 1 byte)
            std::vector<int> v{f.in};
            std::vector<char> in(n.st.size(), 0);
            in[f.in] = 1;
            for (size_t h = 0; h < v.size(); h++)
                for (int y : n.st[v[h]].eps) if (!in[y]) { in[y] = 1; v.push_back(y); }
            if (in[f.out] || len == 0) return "regex: expression matches the empty string (expression " + std::to_string(j) + ")";
        }
        n.st[acc].accept = (int)j;
        n.st[f.out].eps.push_back(acc);
        n.st[start].eps.push_back(f.in);
        o.maxlen = len > REGEX_PAR_MAXLEN ? 0xFFFFFFFFu : std::max(o.maxlen, (uint32_t)len);
    }
    const int ns = (int)n.st.size();
    auto closure = [&](std::vector<int> &v) {
        std::vector<char> in(ns, 0);
        for (int x : v) in[x] = 1;
        for (size_t h = 0; h < v.size(); h++)
            for (int y : n.st[v[h]].eps) if (!in[y]) { in[y] = 1; v.push_back(y); }
        std::sort(v.begin(), v.end());
    };
    std::map<std::vector<int>, uint32_t> id;
    std::vector<std::vector<int>> sets;
    std::vector<int> s0{start};
    closure(s0);
    id[s0] = 0;
    sets.push_back(s0);
    std::vector<uint32_t> delta;
    for (size_t h = 0; h < sets.size(); h++) {
        if (sets.size() > max_states) return "regex: DFA exceeds " + std::to_string(max_states) + " states";
        const std::vector<int> cur = sets[h];
        for (int b = 0; b < 256; b++) {
            std::vector<int> nx{start};
            for (int x : cur)
                if (n.st[x].out >= 0 && (n.st[x].set[b >> 6] >> (b & 63) & 1)) nx.push_back(n.st[x].out);
            closure(nx);
            nx.erase(std::unique(nx.begin(), nx.end()), nx.end());
            auto it = id.find(nx);
            uint32_t t;
            if (it == id.end()) { t = (uint32_t)sets.size(); id.emplace(nx, t); sets.push_back(nx); }
            else t = it->second;
            delta.push_back(t);
        }
    }
    const uint32_t N = (uint32_t)sets.size();
    o.n_states = N;
    o.ncls = 256;
    o.wide = N > 32768 ? 1 : 0;
    o.cls.resize(256);
    for (int b = 0; b < 256; b++) o.cls[b] = (uint8_t)b;
    o.out_off.assign(N + 1, 0);
    o.out_ids.clear();
    std::vector<char> accepting(N, 0);
    for (uint32_t k = 0; k < N; k++) {
        o.out_off[k] = (uint32_t)o.out_ids.size();
        std::vector<uint16_t> ids;
        for (int x : sets[k]) if (n.st[x].accept >= 0) ids.push_back((uint16_t)n.st[x].accept);
        std::sort(ids.begin(), ids.end());
        ids.erase(std::unique(ids.begin(), ids.end()), ids.end());
        accepting[k] = !ids.empty();
        o.out_ids.insert(o.out_ids.end(), ids.begin(), ids.end());
    }
    o.out_off[N] = (uint32_t)o.out_ids.size();
    if (o.out_ids.empty()) o.out_ids.push_back(0);
    const size_t es = o.wide ? 4 : 2;
    o.trans.assign((size_t)N * 256 * es, 0);
    for (size_t k = 0; k < (size_t)N * 256; k++) {
        uint32_t t = delta[k];
        uint32_t e = t | (accepting[t] ? (o.wide ? 0x80000000u : 0x8000u) : 0u);
        if (o.wide) memcpy(&o.trans[k * 4], &e, 4);
        else { uint16_t e16 = (uint16_t)e; memcpy(&o.trans[k * 2], &e16, 2); }
    }
    o.action.assign(s.action, s.action + s.n_patterns);
    return "";
}

}  // namespace nfc
