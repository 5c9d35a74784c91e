// csrc/host/format.cpp — S10 host-side stdout formatting.
//
// Instances write {fmt id, raw 8-byte arguments} records on the device
// (rt/device_rt.cuh ens_printf); the host expands them with the format table
// below, in instance order (reading Q9).  Only exact quantities are printed
// (integers, strings, doubles exact by construction: SURVEY.md §8(c) "Stdout
// rule"), so the bytes equal a CPU run's printf output.
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <string>

#include "../rt/fmt_ids.h"

namespace ens {

static const char *const kFmt[FMT_COUNT] = {
    /* FMT_BADARG    */ "%s: invalid argument '%s'\n",
    /* FMT_USAGE_XS  */
    "usage: %s [-s small|large] [-g gridpoints] [-l lookups] [-G unionized|nuclide|hash] [-h hash_bins] "
    "[-m event|history] [-p particles] [-r seed] [-R grid_seed]\n",
    /* FMT_USAGE_RS  */ "usage: %s [-s small|large] [-l lookups] [-p poles] [-w windows] [-d] [-r seed] [-R init_seed]\n",
    /* FMT_USAGE_AMG */ "usage: %s [-x nx] [-y ny] [-z nz] [-i iters] [-k relax|matvec|both] [-r seed]\n",
    /* FMT_NOTFOUND  */ "%s: command not found\n",
    /* FMT_ECHO_ARGC */ "argc=%d\n",
    /* FMT_ECHO_ARGV */ "argv[%d]=%s\n",
    /* FMT_XS_HDR    */ "XSBench-style HM=%s n_iso=%d n_gp=%ld grid=%s L=%ld seed=%lu\n",
    /* FMT_VERIFY    */ "Verification checksum: %lu\n",
    /* FMT_RS_HDR    */ "RSBench-style HM=%s n_nuc=%d poles=%d windows=%d doppler=%d L=%ld seed=%lu\n",
    /* FMT_AMG       */ "AMGmk-style n=%d nnz=%d iters=%d maxerr=%.17g\n",
    /* FMT_XS_HIST   */ "XSBench-style history HM=%s n_iso=%d n_gp=%ld grid=%s particles=%ld L=%ld seed=%lu\n",
    /* FMT_USAGE_PR  */ "usage: %s [-n nodes] [-e avg_degree] [-i iterations] [-R graph_seed]\n",
    /* FMT_PR        */ "PageRank-style n=%ld edges=%ld iters=%ld top=%ld\n",
};

// Expand one format with its slots; returns false on malformed input.
static bool expand(const char *fmt, const uint64_t *slots, size_t nslots, std::string &out) {
  size_t si = 0;
  char spec[64], buf[512];
  for (const char *p = fmt; *p;) {
    if (*p != '%') {
      out.push_back(*p++);
      continue;
    }
    if (p[1] == '%') {
      out.push_back('%');
      p += 2;
      continue;
    }
    // %[flags][width][.prec][length]conv
    const char *q = p + 1;
    std::string head = "%";
    while (*q && std::strchr("-+ #0", *q)) head.push_back(*q++);
    while (*q >= '0' && *q <= '9') head.push_back(*q++);
    if (*q == '.') {
      head.push_back(*q++);
      while (*q >= '0' && *q <= '9') head.push_back(*q++);
    }
    while (*q == 'l' || *q == 'h' || *q == 'z') q++;
    const char conv = *q;
    if (!conv) return false;
    if (si >= nslots) return false;
    int k = 0;
    switch (conv) {
      case 'd': case 'i':
        std::snprintf(spec, sizeof spec, "%slld", head.c_str());
        k = std::snprintf(buf, sizeof buf, spec, (long long)slots[si++]);
        break;
      case 'u': case 'x': case 'X': case 'o':
        std::snprintf(spec, sizeof spec, "%sll%c", head.c_str(), conv);
        k = std::snprintf(buf, sizeof buf, spec, (unsigned long long)slots[si++]);
        break;
      case 'g': case 'f': case 'e': case 'G': case 'E': {
        double d;
        std::memcpy(&d, &slots[si++], 8);
        std::snprintf(spec, sizeof spec, "%s%c", head.c_str(), conv);
        k = std::snprintf(buf, sizeof buf, spec, d);
        break;
      }
      case 's': {
        const uint64_t len = slots[si++];
        const size_t words = (size_t)((len + 7) / 8);
        if (si + words > nslots) return false;
        std::string s((const char *)&slots[si], (size_t)len);
        si += words;
        std::snprintf(spec, sizeof spec, "%ss", head.c_str());
        k = std::snprintf(buf, sizeof buf, spec, s.c_str());
        if (k >= (int)sizeof buf) {  // long strings: no width handling needed
          out += s;
          k = 0;
        }
        break;
      }
      default:
        return false;
    }
    if (k > 0) out.append(buf, (size_t)k < sizeof buf ? (size_t)k : sizeof buf - 1);
    p = q + 1;
  }
  return true;
}

// raw: sequence of records {u32 fmt, u32 payload bytes, payload}
long format_raw(const void *raw, size_t raw_len, std::string &out) {
  const unsigned char *b = (const unsigned char *)raw;
  size_t off = 0;
  while (off + 8 <= raw_len) {
    uint64_t hdr;
    std::memcpy(&hdr, b + off, 8);
    const uint32_t fmt = (uint32_t)(hdr & 0xffffffffu), payload = (uint32_t)(hdr >> 32);
    if (fmt >= FMT_COUNT || payload % 8 || off + 8 + payload > raw_len) return -1;
    const uint64_t *slots = (const uint64_t *)(b + off + 8);
    if (!expand(kFmt[fmt], slots, payload / 8, out)) return -1;
    off += 8 + payload;
  }
  return off == raw_len ? (long)out.size() : -1;
}

}  // namespace ens
