// plan.cpp — parser for plan segments (grammar in DESIGN.md §4).
#include "plan.h"

#include <cctype>
#include <climits>
#include <sstream>

#include "common.h"

namespace gpl {
namespace {

struct Tok {
  enum K { ID, INT, SYM, END } k;
  std::string s;
  int64_t v = 0;
};

bool tokenize(const std::string& line, std::vector<Tok>* out, std::string* err) {
  size_t i = 0, n = line.size();
  while (i < n) {
    char c = line[i];
    if (c == '#') break;
    if (std::isspace((unsigned char)c)) { i++; continue; }
    if (std::isalpha((unsigned char)c) || c == '_') {
      size_t j = i;
      while (j < n && (std::isalnum((unsigned char)line[j]) || line[j] == '_')) j++;
      out->push_back({Tok::ID, line.substr(i, j - i)});
      i = j;
      continue;
    }
    bool neg_num = (c == '-' && i + 1 < n && std::isdigit((unsigned char)line[i + 1]) &&
                    (out->empty() || (out->back().k == Tok::SYM && out->back().s != ")")));
    if (std::isdigit((unsigned char)c) || neg_num) {
      size_t j = i + (neg_num ? 1 : 0);
      while (j < n && std::isdigit((unsigned char)line[j])) j++;
      Tok t{Tok::INT, line.substr(i, j - i)};
      try {
        t.v = std::stoll(t.s);
      } catch (...) {
        *err = "integer out of range: " + t.s;
        return false;
      }
      out->push_back(t);
      i = j;
      continue;
    }
    static const char* two[] = {"->", "==", "!=", "<=", ">="};
    bool matched = false;
    for (const char* s : two) {
      if (line.compare(i, 2, s) == 0) {
        out->push_back({Tok::SYM, s});
        i += 2;
        matched = true;
        break;
      }
    }
    if (matched) continue;
    if (std::string("{}(),<>*-+/").find(c) != std::string::npos) {
      out->push_back({Tok::SYM, std::string(1, c)});
      i++;
      continue;
    }
    *err = std::string("unexpected character '") + c + "'";
    return false;
  }
  out->push_back({Tok::END, ""});
  return true;
}

struct Cursor {
  std::vector<Tok> t;
  size_t i = 0;
  const Tok& peek() const { return t[i]; }
  bool is_sym(const char* s) const { return t[i].k == Tok::SYM && t[i].s == s; }
  bool is_id(const char* s) const { return t[i].k == Tok::ID && t[i].s == s; }
  bool accept_sym(const char* s) {
    if (is_sym(s)) { i++; return true; }
    return false;
  }
};

struct ParseError {
  std::string msg;
};

std::string expect_id(Cursor& c, const char* what) {
  if (c.peek().k != Tok::ID) throw ParseError{std::string("expected ") + what};
  return c.t[c.i++].s;
}
int64_t expect_int(Cursor& c, const char* what) {
  if (c.peek().k != Tok::INT) throw ParseError{std::string("expected integer ") + what};
  return c.t[c.i++].v;
}
void expect_sym(Cursor& c, const char* s) {
  if (!c.accept_sym(s)) throw ParseError{std::string("expected '") + s + "'"};
}
void expect_end(Cursor& c) {
  if (c.peek().k != Tok::END) throw ParseError{"unexpected trailing token '" + c.peek().s + "'"};
}

// KEYSPEC: COL | (COL, COL)
std::vector<std::string> parse_keys(Cursor& c) {
  std::vector<std::string> k;
  if (c.accept_sym("(")) {
    k.push_back(expect_id(c, "key column"));
    expect_sym(c, ",");
    k.push_back(expect_id(c, "key column"));
    expect_sym(c, ")");
  } else {
    k.push_back(expect_id(c, "key column"));
  }
  return k;
}

// REF: NAME | year(NAME)
RefIR parse_ref(Cursor& c) {
  RefIR r;
  std::string id = expect_id(c, "column or slot");
  if (id == "year" && c.is_sym("(")) {
    c.i++;
    r.kind = RefIR::YEARCOL;
    r.name = expect_id(c, "date column");
    expect_sym(c, ")");
  } else {
    r.kind = RefIR::COL;  // resolved to SLOT later if it names a slot
    r.name = id;
  }
  return r;
}

// Comparison tail shared by filter and where: OP ...  -> (kind, lo, hi, mask)
void parse_cmp(Cursor& c, int* kind, int64_t* lo, int64_t* hi, uint64_t* mask) {
  *kind = F_RANGE;
  *lo = INT64_MIN;
  *hi = INT64_MAX;
  *mask = 0;
  if (c.is_id("between")) {
    c.i++;
    *lo = expect_int(c, "lower bound");
    expect_id(c, "'and'");
    *hi = expect_int(c, "upper bound");
  } else if (c.is_id("in")) {
    c.i++;
    expect_sym(c, "{");
    *kind = F_MASK;
    do {
      int64_t v = expect_int(c, "set member");
      if (v < 0 || v > 63) throw ParseError{"'in' set members must be in [0, 63]"};
      *mask |= 1ull << v;
    } while (c.accept_sym(","));
    expect_sym(c, "}");
  } else if (c.accept_sym("==")) {
    *lo = *hi = expect_int(c, "constant");
  } else if (c.accept_sym("!=")) {
    *kind = F_NE;
    *lo = expect_int(c, "constant");
  } else if (c.accept_sym("<=")) {
    *hi = expect_int(c, "constant");
  } else if (c.accept_sym(">=")) {
    *lo = expect_int(c, "constant");
  } else if (c.accept_sym("<")) {
    int64_t v = expect_int(c, "constant");
    if (v == INT64_MIN) throw ParseError{"empty range"};
    *hi = v - 1;
  } else if (c.accept_sym(">")) {
    int64_t v = expect_int(c, "constant");
    if (v == INT64_MAX) throw ParseError{"empty range"};
    *lo = v + 1;
  } else {
    throw ParseError{"expected comparison (between/in/==/!=/</<=/>/>=)"};
  }
}

// FACTOR: NAME | INT | ( INT (+|-) NAME ) | ( NAME )
FactorIR parse_factor(Cursor& c) {
  FactorIR f;
  if (c.peek().k == Tok::INT) {
    f.x.kind = RefIR::CONST;
    f.a = c.t[c.i++].v;
    f.b = 0;
    return f;
  }
  if (c.accept_sym("(")) {
    if (c.peek().k == Tok::INT) {
      f.a = c.t[c.i++].v;
      if (c.accept_sym("-")) f.b = -1;
      else if (c.accept_sym("+")) f.b = 1;
      else throw ParseError{"expected '+' or '-' in (const +/- column)"};
    } else {
      f.a = 0;
      f.b = 1;
    }
    f.x.kind = RefIR::COL;
    f.x.name = expect_id(c, "column or slot");
    expect_sym(c, ")");
    return f;
  }
  f.x.kind = RefIR::COL;
  f.x.name = expect_id(c, "column or slot");
  f.a = 0;
  f.b = 1;
  return f;
}

std::vector<TermIR> parse_value(Cursor& c) {
  std::vector<TermIR> terms;
  int sign = 1;
  for (;;) {
    TermIR t;
    t.sign = sign;
    t.f.push_back(parse_factor(c));
    while (c.accept_sym("*")) t.f.push_back(parse_factor(c));
    if ((int)t.f.size() > MAXFACT) throw ParseError{"too many factors in a term"};
    terms.push_back(t);
    if (c.accept_sym("-")) sign = -1;
    else if (c.accept_sym("+")) sign = 1;
    else break;
  }
  if ((int)terms.size() > MAXTERM) throw ParseError{"value has too many terms"};
  return terms;
}

}  // namespace

bool parse_segment(const std::string& text, Segment* seg, std::string* err) {
  *seg = Segment();
  seg->text = text;
  std::istringstream in(text);
  std::string line;
  int lineno = 0;
  bool have_head = false;
  seg->aggs.push_back(AggIR{A_COUNT, "", 0});
  try {
    while (std::getline(in, line)) {
      lineno++;
      Cursor c;
      std::string terr;
      if (!tokenize(line, &c.t, &terr)) throw ParseError{terr};
      if (c.peek().k == Tok::END) continue;
      std::string kw = expect_id(c, "statement keyword");
      if (!have_head) {
        if (kw == "build") {
          seg->is_build = true;
          seg->name = expect_id(c, "hash table name");
          expect_end(c);
        } else if (kw == "run") {
          seg->is_build = false;
          seg->table = expect_id(c, "table name");
          expect_end(c);
        } else if (kw == "partition") {
          // a blocking segment like a build ("the partition phase"), with a table as output
          seg->is_build = true;
          seg->is_partition = true;
          seg->name = expect_id(c, "partitioned table name");
          expect_end(c);
        } else {
          throw ParseError{"segment must start with 'build NAME', 'partition NAME' or 'run TABLE'"};
        }
        have_head = true;
        continue;
      }
      if (kw == "scan") {
        if (!seg->is_build) throw ParseError{"'scan' only in build segments (use 'run TABLE')"};
        seg->table = expect_id(c, "table name");
      } else if (kw == "filter") {
        FilterIR f;
        f.col = expect_id(c, "column");
        parse_cmp(c, &f.kind, &f.lo, &f.hi, &f.mask);
        seg->filters.push_back(f);
      } else if (kw == "probe" || kw == "semi" || kw == "mark") {
        ProbeIR p;
        p.kind = kw == "probe" ? P_INNER : kw == "semi" ? P_SEMI : P_MARK;
        p.ht = expect_id(c, "hash table name");
        p.keys = parse_keys(c);
        if (c.accept_sym("->")) p.out = expect_id(c, "slot name");
        if (p.kind == P_MARK && p.out.empty()) throw ParseError{"'mark' needs '-> flag'"};
        if (p.kind == P_SEMI && !p.out.empty()) throw ParseError{"'semi' takes no output slot"};
        seg->probes.push_back(p);
      } else if (kw == "key") {
        if (!seg->is_build) throw ParseError{"'key' only in build segments"};
        seg->key = parse_keys(c);
        if (seg->is_partition) {
          if (expect_id(c, "by") != "by") throw ParseError{"partition key needs 'by HT'"};
          seg->by_ht = expect_id(c, "hash table");
          if (seg->key.size() != 1) throw ParseError{"partition key is one column"};
        }
      } else if (kw == "parts") {
        if (!seg->is_partition) throw ParseError{"'parts' only in partition segments"};
        const int64_t P = expect_int(c, "partition count");
        if (P < 2 || P > 4096 || (P & (P - 1))) throw ParseError{"parts: a power of two in [2, 4096]"};
        seg->nparts = (int)P;
      } else if (kw == "payload") {
        if (!seg->is_build || seg->is_partition) throw ParseError{"'payload' only in build segments"};
        seg->payload = parse_ref(c);
      } else if (kw == "hash") {
        std::string h = expect_id(c, "auto|direct|mult|ordered");
        if (h == "mult") seg->hash = H_MULT;
        else if (h == "ordered") seg->hash = H_ORDERED;
        else if (h == "direct") seg->hash = 2;
        else if (h == "auto") seg->hash = -1;
        else throw ParseError{"hash must be auto, direct, mult or ordered"};
      } else if (kw == "multi") {  // non-unique key: every match joins (NEXT-4 fan-out)
        if (!seg->is_build || seg->is_partition) throw ParseError{"'multi' only in build segments"};
        seg->multi = true;
      } else if (kw == "load") {
        seg->load_pct = (int)expect_int(c, "percent");
        if (seg->load_pct < 10 || seg->load_pct > 90) throw ParseError{"load must be in [10, 90]"};
      } else if (kw == "where") {
        if (seg->is_build) throw ParseError{"'where' only in the probe segment"};
        WhereIR w;
        if (c.accept_sym("(")) {
          w.kind = R_PAIRS;
          w.a = expect_id(c, "slot");
          expect_sym(c, ",");
          w.b = expect_id(c, "slot");
          expect_sym(c, ")");
          if (!c.is_id("in")) throw ParseError{"expected 'in'"};
          c.i++;
          expect_sym(c, "{");
          do {
            expect_sym(c, "(");
            int64_t x = expect_int(c, "pair member");
            expect_sym(c, ",");
            int64_t y = expect_int(c, "pair member");
            expect_sym(c, ")");
            w.pairs.push_back({x, y});
          } while (c.accept_sym(","));
          expect_sym(c, "}");
          if (w.pairs.size() > 4) throw ParseError{"at most 4 pairs"};
        } else {
          w.a = expect_id(c, "slot");
          if (c.is_sym("==") && c.t[c.i + 1].k == Tok::ID) {
            c.i++;
            w.kind = R_EQ;
            w.b = expect_id(c, "slot");
          } else {
            int kind;
            parse_cmp(c, &kind, &w.lo, &w.hi, &w.mask);
            w.kind = kind == F_MASK ? R_MASK : kind == F_RANGE ? R_RANGE : -1;
            if (w.kind < 0) throw ParseError{"'!=' not supported in where"};
          }
        }
        seg->wheres.push_back(w);
      } else if (kw == "group" && c.is_id("hash")) {
        // hash group-by over unbounded int32 keys: group hash A[, B]
        if (seg->is_build) throw ParseError{"'group' only in the probe segment"};
        if (!seg->groups.empty()) throw ParseError{"one 'group hash' statement, not mixed with dense groups"};
        c.i++;
        seg->hash_group = true;
        do {
          GroupIR g;
          g.ref = parse_ref(c);
          seg->groups.push_back(g);
        } while (c.accept_sym(","));
        if (seg->groups.size() > 2) throw ParseError{"group hash takes at most 2 keys"};
      } else if (kw == "order") {
        if (seg->is_build) throw ParseError{"'order' only in the probe segment"};
        do {
          OrderIR o;
          std::string what = expect_id(c, "agg|key");
          if (what != "agg" && what != "key") throw ParseError{"order component must be 'agg N' or 'key N'"};
          o.is_agg = what == "agg";
          o.idx = (int)expect_int(c, "index");
          if (c.is_id("desc") || c.is_id("asc")) {
            o.desc = c.is_id("desc");
            c.i++;
          }
          seg->order.push_back(o);
        } while (c.accept_sym(","));
        if (seg->order.size() > 3) throw ParseError{"at most 3 order components"};
      } else if (kw == "decode") {
        // decode key I TABLE KEYCOL -> OUTCOL (A10: e.g. nation key -> n_name)
        if (seg->is_build) throw ParseError{"'decode' only in the probe segment"};
        if (expect_id(c, "key") != "key") throw ParseError{"decode needs 'key N'"};
        DecodeIR dc;
        dc.key = (int)expect_int(c, "key index");
        dc.table = expect_id(c, "table");
        dc.keycol = expect_id(c, "key column");
        expect_sym(c, "->");
        dc.outcol = expect_id(c, "output column");
        seg->decodes.push_back(dc);
      } else if (kw == "ratio") {
        // ratio [C *] agg I / agg J   (A10: Q8 mkt_share, Q14 promo_revenue)
        if (seg->is_build) throw ParseError{"'ratio' only in the probe segment"};
        RatioIR r;
        if (c.t[c.i].k == Tok::INT) {
          r.scale = (double)expect_int(c, "scale");
          expect_sym(c, "*");
        }
        if (expect_id(c, "agg") != "agg") throw ParseError{"ratio operands are 'agg N'"};
        r.num = (int)expect_int(c, "agg index");
        expect_sym(c, "/");
        if (expect_id(c, "agg") != "agg") throw ParseError{"ratio operands are 'agg N'"};
        r.den = (int)expect_int(c, "agg index");
        seg->ratios.push_back(r);
      } else if (kw == "limit") {
        if (seg->is_build) throw ParseError{"'limit' only in the probe segment"};
        const int64_t k = expect_int(c, "row count");
        if (k < 1 || k > 512) throw ParseError{"limit must be in [1, 512]"};
        seg->limit = (int)k;
      } else if (kw == "group") {
        if (seg->is_build) throw ParseError{"'group' only in the probe segment"};
        if (seg->hash_group) throw ParseError{"dense groups cannot follow 'group hash'"};
        GroupIR g;
        g.ref = parse_ref(c);
        g.lo = expect_int(c, "domain lower bound");
        g.hi = expect_int(c, "domain upper bound (exclusive)");
        if (g.hi <= g.lo) throw ParseError{"empty group domain"};
        seg->groups.push_back(g);
      } else if (kw == "value") {
        if (seg->is_build) throw ParseError{"'value' only in the probe segment"};
        seg->value = parse_value(c);
      } else if (kw == "agg") {
        if (seg->is_build) throw ParseError{"'agg' only in the probe segment"};
        std::string f = expect_id(c, "count|sum");
        if (f == "count") {
          // COUNT(*) is always aggregate 0
        } else if (f == "sum") {
          AggIR a{A_SUM, "", 0};
          if (c.is_id("if")) {
            c.i++;
            a.slot = expect_id(c, "slot");
            if (c.accept_sym("==")) {
              a.kind = A_SUMIFEQ;
              a.c = expect_int(c, "constant");
            } else {
              a.kind = A_SUMIF;
            }
          }
          seg->aggs.push_back(a);
        } else {
          throw ParseError{"agg must be 'count' or 'sum [if SLOT [== C]]'"};
        }
      } else if (kw == "split") {
        seg->split_hint = (int)expect_int(c, "probe count");
      } else {
        throw ParseError{"unknown statement '" + kw + "'"};
      }
      expect_end(c);
    }
    if (!have_head) throw ParseError{"empty segment"};
    if (seg->table.empty()) throw ParseError{"no scanned table"};
    if (seg->is_build && seg->key.empty()) throw ParseError{"build segment needs 'key'"};
    if (!seg->is_build && (int)seg->aggs.size() > MAXA) throw ParseError{"too many aggregates"};
    if ((int)seg->filters.size() > MAXF) throw ParseError{"too many filters"};
    if ((int)seg->probes.size() > MAXP) throw ParseError{"too many probes"};
    if ((int)seg->wheres.size() > MAXR) throw ParseError{"too many where clauses"};
    if ((int)seg->groups.size() > MAXG) throw ParseError{"too many group dimensions"};
    for (auto& dc : seg->decodes)
      if (dc.key < 0 || dc.key >= (int)seg->groups.size() || seg->hash_group)
        throw ParseError{"decode: key index out of range (dense group keys only)"};
    if (seg->ratios.size() > 2) throw ParseError{"at most 2 ratio columns"};
    for (auto& r : seg->ratios)
      if (r.num < 0 || r.den < 0 || r.num >= (int)seg->aggs.size() || r.den >= (int)seg->aggs.size())
        throw ParseError{"ratio: agg index out of range"};
    if (seg->limit && seg->order.empty()) throw ParseError{"'limit' needs an 'order' statement"};
    for (auto& o : seg->order)
      if (o.idx < 0 || (o.is_agg ? o.idx >= (int)seg->aggs.size() : o.idx >= (int)seg->groups.size()))
        throw ParseError{"order component index out of range"};
    bool has_sum = false;
    for (auto& a : seg->aggs) has_sum |= a.kind != A_COUNT;
    if (has_sum && seg->value.empty()) throw ParseError{"'agg sum' needs a 'value' statement"};
  } catch (const ParseError& e) {
    *err = "plan line " + std::to_string(lineno) + ": " + e.msg;
    return false;
  }
  return true;
}

}  // namespace gpl
