// format.cpp -- tracePrint's textual / CSV output, laid out
// like Fig. 4.  Host-only, no GPU.
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include <string>

#include "xpl.h"

namespace {

std::string name_of(const xpl_alloc_report& r, const xpl_name* names, size_t n_names) {
  if (r.name_idx != 0xFFFFFFFFu && r.name_idx < n_names && names && names[r.name_idx].expr &&
      names[r.name_idx].expr[0])
    return names[r.name_idx].expr;
  char b[64];
  snprintf(b, sizeof b, "alloc %llu", (unsigned long long)r.id);
  return b;
}

void add(std::string& o, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
void add(std::string& o, const char* fmt, ...) {
  char b[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(b, sizeof b, fmt, ap);
  va_end(ap);
  o += b;
}

}  // namespace

extern "C" xpl_status xpl_format_reports(const xpl_alloc_report* reps, size_t n,
                                         const xpl_name* names, size_t n_names, int csv,
                                         int only_named, char* buf, size_t cap, size_t* needed) {
  if ((!reps && n) || !needed || (!buf && cap)) return XPL_ERR_INVALID_ARG;
  std::string o;
  size_t shown = 0;
  for (size_t i = 0; i < n; ++i)
    if (!only_named || reps[i].name_idx != 0xFFFFFFFFu) ++shown;
  if (csv) {
    o += "id,name,base,bytes,words,kind,live,w_c,w_g,r_cc,r_cg,r_gc,r_gg,any_acc,gpu_acc,"
         "alternating,density_pct_any,density_pct_gpu,low_density_blocks,low_density_words,"
         "h2d_unused_runs,h2d_unused_words,d2h_unneeded_runs,d2h_unneeded_words,ever_accessed,flags\n";
  } else {
    add(o, "*** checking %zu %sallocations\n", shown, only_named ? "named " : "");
  }
  for (size_t i = 0; i < n; ++i) {
    const xpl_alloc_report& r = reps[i];
    if (only_named && r.name_idx == 0xFFFFFFFFu) continue;
    const std::string nm = name_of(r, names, n_names);
    if (csv) {
      add(o, "%llu,\"%s\",%llu,%llu,%llu,%u,%u,%llu,%llu,%llu,%llu,%llu,%llu,%llu,%llu,%llu,%llu,%llu,"
             "%llu,%llu,%llu,%llu,%llu,%llu,%llu,%u\n",
          (unsigned long long)r.id, nm.c_str(), (unsigned long long)r.base, (unsigned long long)r.bytes,
          (unsigned long long)r.words, r.kind, r.live, (unsigned long long)r.w_c,
          (unsigned long long)r.w_g, (unsigned long long)r.r_cc, (unsigned long long)r.r_cg,
          (unsigned long long)r.r_gc, (unsigned long long)r.r_gg, (unsigned long long)r.any_acc,
          (unsigned long long)r.gpu_acc, (unsigned long long)r.alternating,
          (unsigned long long)r.density_pct_any, (unsigned long long)r.density_pct_gpu,
          (unsigned long long)r.low_density_blocks, (unsigned long long)r.low_density_words,
          (unsigned long long)r.h2d_unused_runs, (unsigned long long)r.h2d_unused_words,
          (unsigned long long)r.d2h_unneeded_runs, (unsigned long long)r.d2h_unneeded_words,
          (unsigned long long)r.ever_accessed, r.flags);
      continue;
    }
    add(o, "%s%s\n", nm.c_str(), r.live ? "" : "  (freed)");
    add(o, "%-18s %-38s\n", "write counts", "write>read counts");
    add(o, "%8s %8s %10s %9s %9s %9s\n", "C", "G", "C>C", "C>G", "G>C", "G>G");
    add(o, "%8llu %8llu %10llu %9llu %9llu %9llu\n", (unsigned long long)r.w_c,
        (unsigned long long)r.w_g, (unsigned long long)r.r_cc, (unsigned long long)r.r_cg,
        (unsigned long long)r.r_gc, (unsigned long long)r.r_gg);
    add(o, "access density (in %%): %llu\n", (unsigned long long)r.density_pct_gpu);
    add(o, "%llu elements with alternating accesses\n", (unsigned long long)r.alternating);
    if (r.flags & XPL_PAT_ALTERNATING) add(o, "  ! alternating CPU/GPU accesses in managed memory\n");
    if (r.flags & XPL_PAT_LOW_DENSITY)
      add(o, "  ! low access density: %llu block(s), %llu words\n",
          (unsigned long long)r.low_density_blocks, (unsigned long long)r.low_density_words);
    if (r.flags & XPL_PAT_UNNEEDED_H2D)
      add(o, "  ! transferred to the GPU but not used there: %llu run(s), %llu words\n",
          (unsigned long long)r.h2d_unused_runs, (unsigned long long)r.h2d_unused_words);
    if (r.flags & XPL_PAT_UNNEEDED_D2H)
      add(o, "  ! transferred back without being updated on the GPU: %llu run(s), %llu words\n",
          (unsigned long long)r.d2h_unneeded_runs, (unsigned long long)r.d2h_unneeded_words);
    if (r.flags & XPL_PAT_UNUSED) add(o, "  ! allocated but not accessed\n");
  }
  *needed = o.size() + 1;
  if (cap < o.size() + 1) return XPL_ERR_INVALID_ARG;
  memcpy(buf, o.c_str(), o.size() + 1);
  return XPL_OK;
}
