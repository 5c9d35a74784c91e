// csrc/rt/fmt_ids.h — stdout format ids (device side writes {fmt_id, raw
// 8-byte arguments}; the host formats them with the table in
// host/format.cpp).  This replaces the paper's host-RPC printf (Fig. 2
// P:247-248): no device->host call happens during a launch, and
// every instance's stdout is a private buffer concatenated in instance order
// (reading Q9).
#pragma once

namespace ens {
enum FmtId : unsigned {
  FMT_BADARG = 0,     // "%s: invalid argument '%s'\n"
  FMT_USAGE_XS = 1,   // xsbench usage line
  FMT_USAGE_RS = 2,   // rsbench usage line
  FMT_USAGE_AMG = 3,  // amgmk usage line
  FMT_NOTFOUND = 4,   // "%s: command not found\n"
  FMT_ECHO_ARGC = 5,  // "argc=%d\n"
  FMT_ECHO_ARGV = 6,  // "argv[%d]=%s\n"
  FMT_XS_HDR = 7,     // XSBench-style header line
  FMT_VERIFY = 8,     // "Verification checksum: %lu\n"
  FMT_RS_HDR = 9,     // RSBench-style header line
  FMT_AMG = 10,       // AMGmk-style result line
  FMT_XS_HIST = 11,   // XSBench-style history-mode header line
  FMT_USAGE_PR = 12,  // pagerank usage line
  FMT_PR = 13,        // Page-Rank-style result line
  FMT_COUNT = 14
};
}  // namespace ens
