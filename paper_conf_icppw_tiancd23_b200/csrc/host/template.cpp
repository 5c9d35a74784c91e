// csrc/host/template.cpp — args-file templating.
//
// The paper plans "a script language specifically for the command line
// argument file ... [to] enable the generation of command line arguments for
// each instance dynamically" (§3.2, future work P:646-648).  This
// is that language, kept small: a line
//
//     @repeat N <template>
//
// expands to N instance lines, i = 0..N-1, where the template's
//     {expr}    is an integer expression in i: + - * / % ( ) and literals
//               (C semantics, left to right within a precedence level), and
//     {a|b|c}   is the (i mod 3)-th alternative.
// Every other line is copied unchanged, so plain args files are unaffected.
#include <cctype>
#include <cstdlib>
#include <cstring>
#include <string>

#include "../../../include/ens.h"

namespace {

struct Expr {
  const char *p, *end;
  long long i;
  bool ok = true;

  void ws() {
    while (p < end && (*p == ' ' || *p == '\t')) p++;
  }
  long long factor() {
    ws();
    if (p >= end) return ok = false, 0;
    if (*p == '(') {
      p++;
      long long v = expr();
      ws();
      if (p >= end || *p != ')') return ok = false, 0;
      p++;
      return v;
    }
    if (*p == '-') {
      p++;
      return -factor();
    }
    if (*p == 'i') {
      p++;
      return i;
    }
    if (std::isdigit((unsigned char)*p)) {
      long long v = 0;
      int nd = 0;
      while (p < end && std::isdigit((unsigned char)*p)) {
        if (++nd > 18) return ok = false, 0;
        v = v * 10 + (*p++ - '0');
      }
      return v;
    }
    return ok = false, 0;
  }
  long long term() {
    long long v = factor();
    for (;;) {
      ws();
      if (p >= end || (*p != '*' && *p != '/' && *p != '%')) return v;
      const char op = *p++;
      const long long r = factor();
      if (op == '*') v *= r;
      else if (r == 0) return ok = false, 0;
      else if (op == '/') v /= r;
      else v %= r;
    }
  }
  long long expr() {
    long long v = term();
    for (;;) {
      ws();
      if (p >= end || (*p != '+' && *p != '-')) return v;
      const char op = *p++;
      const long long r = term();
      v = op == '+' ? v + r : v - r;
    }
  }
};

// expand one template for index i; false on a malformed placeholder
bool expand_one(const std::string &tpl, long long i, std::string &out) {
  size_t k = 0;
  while (k < tpl.size()) {
    if (tpl[k] != '{') {
      out.push_back(tpl[k++]);
      continue;
    }
    const size_t close = tpl.find('}', k);
    if (close == std::string::npos) return false;
    const std::string body = tpl.substr(k + 1, close - k - 1);
    if (body.find('|') != std::string::npos) {  // choice
      size_t n = 1;
      for (char ch : body) n += ch == '|';
      long long sel = i % (long long)n;
      if (sel < 0) sel += (long long)n;
      size_t s = 0;
      for (long long a = 0; a < sel; a++) s = body.find('|', s) + 1;
      const size_t e = body.find('|', s);
      out += body.substr(s, e == std::string::npos ? std::string::npos : e - s);
    } else {
      Expr x{body.data(), body.data() + body.size(), i};
      const long long v = x.expr();
      x.ws();
      if (!x.ok || x.p != x.end) return false;
      out += std::to_string(v);
    }
    k = close + 1;
  }
  return true;
}

}  // namespace

namespace ens {
// Expand `text`; returns ENS_OK, or ENS_EPARSE with *bad_line = 0-based line.
int expand_args(const char *text, size_t len, std::string &out, long *bad_line) {
  out.clear();
  size_t pos = 0;
  long line_no = 0;
  while (pos < len) {
    const char *nl = (const char *)std::memchr(text + pos, '\n', len - pos);
    const size_t end = nl ? (size_t)(nl - text) : len;
    std::string line(text + pos, end - pos);
    if (line.rfind("@repeat", 0) == 0 && (line.size() == 7 || line[7] == ' ' || line[7] == '\t')) {
      size_t k = 7;
      while (k < line.size() && (line[k] == ' ' || line[k] == '\t')) k++;
      size_t s = k;
      while (k < line.size() && std::isdigit((unsigned char)line[k])) k++;
      if (k == s || k - s > 8) {
        *bad_line = line_no;
        return ENS_EPARSE;
      }
      const long long n = std::atoll(line.substr(s, k - s).c_str());
      while (k < line.size() && (line[k] == ' ' || line[k] == '\t')) k++;
      std::string tpl = line.substr(k);
      if (!tpl.empty() && tpl.back() == '\r') tpl.pop_back();
      for (long long i = 0; i < n; i++) {
        if (!expand_one(tpl, i, out)) {
          *bad_line = line_no;
          return ENS_EPARSE;
        }
        out.push_back('\n');
      }
    } else {
      out.append(line);
      if (nl) out.push_back('\n');
    }
    if (!nl) break;
    pos = end + 1;
    line_no++;
  }
  return ENS_OK;
}
}  // namespace ens

extern "C" long ens_expand_args(const char *text, size_t len, char *out, size_t cap) {
  if (!text && len) return ENS_EINVAL;
  std::string s;
  long bad = -1;
  const int rc = ens::expand_args(text, len, s, &bad);
  if (rc) return rc;
  if (out) std::memcpy(out, s.data(), s.size() < cap ? s.size() : cap);
  return (long)s.size();
}
