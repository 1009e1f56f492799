// vp_tune.cu — the VersaPipe auto-tuner (§7, Fig. 10) and config
// (de)serialisation.
//
// Fig. 10:  for g in groupings: for s in SM mappings(g): for b in block mappings(s):
//             newtime = timeoutexec(mintime, {g, s, b}); keep the minimum.
// Pruning (L45): "a stage can only be grouped with its neighbouring stages"; per group the
// models RTC, KBK, Megakernel and fine pipeline; per-stage block counts bounded by the
// profiled maximum and equal on every assigned SM (the runtime's greedy fine quotas).
// B200 additions: 148 SMs instead of the paper's 13/20, so the SM
// mapping is searched in two phases — (1) every grouping x model assignment with an SM
// split proportional to the profiled per-stage work (in-kernel %globaltimer accumulators
// of a megakernel run), (2) around the best few, every split at the SM granularity (two
// groups) or a +/- neighbourhood (more groups), and the batch choices.  The timeout is
// enforced on the device by the run watchdog (and by the host for wave-driven groups).
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <string>
#include <vector>

#include "../../include/vp.h"

extern "C" {  // internal accessors defined in vp_host.cu (not part of vp.h)
int vpi_num_stages(void* h);
int vpi_num_sms(void* h);
int vpi_rtc_legal(void* h, int lo, int hi);
int vpi_default_batch(void* h, int s);
uint32_t vpi_swap_flags(void* h, uint32_t flags);
double vpi_timeout(void* h);
void vpi_set_error(void* h, const char* msg);
}

namespace {

struct Shape {      // a grouping with per-group models and an SM split
  int G;
  int lo[VP_MAX_STAGES], hi[VP_MAX_STAGES], gm[VP_MAX_STAGES], sms[VP_MAX_STAGES];
  int div;          // batch divisor
};

void set_range(uint32_t* mask, int a, int b) {
  for (int i = a; i < b && i < VP_MAX_SM; ++i) mask[i >> 5] |= 1u << (i & 31);
}

vp_config to_config(void* p, int S, const Shape& sh) {
  vp_config c;
  memset(&c, 0, sizeof(c));
  c.model = VP_HYBRID;
  c.has_binding = 1;
  c.binding.num_groups = sh.G;
  int start = 0;
  for (int g = 0; g < sh.G; ++g) {
    for (int s = sh.lo[g]; s <= sh.hi[g]; ++s) c.binding.group_of_stage[s] = g;
    c.binding.group_model[g] = sh.gm[g];
    set_range(c.binding.group_sm_mask[g], start, start + sh.sms[g]);
    start += sh.sms[g];
  }
  for (int s = 0; s < S; ++s) c.binding.batch[s] = std::max(1, vpi_default_batch(p, s) / std::max(1, sh.div));
  return c;
}

// timeoutexec(mintime, config): configure, one warm run with a generous limit, then
// `reps` runs with the watchdog at `limit_ms`; best device ms, or < 0 (invalid / timeout).
// A CUDA error (e.g. an illegal address) is sticky for the context: *fatal is set and
// the search stops instead of ranking the remaining candidates on a dead context.
double timeoutexec(void* p, const vp_config& c, double limit_ms, int reps, bool* timed_out, vp_status* fatal) {
  *timed_out = false;
  if (vp_configure_config(p, &c) != VP_OK) return -1.0;
  vp_run_stats st;
  vp_set_timeout(p, std::max(50.0, 4.0 * limit_ms));
  vp_status rc = vp_run(p, nullptr, &st);
  if (rc != VP_OK) {
    *timed_out = rc == VP_ERR_TIMEOUT;
    if (rc == VP_ERR_CUDA) *fatal = rc;
    return -1.0;
  }
  double best = 1e30;
  vp_set_timeout(p, std::max(0.05, limit_ms));
  for (int r = 0; r < reps; ++r) {
    rc = vp_run(p, nullptr, &st);
    if (rc != VP_OK) {
      *timed_out = rc == VP_ERR_TIMEOUT;
      if (rc == VP_ERR_CUDA) *fatal = rc;
      return -1.0;
    }
    best = std::min(best, st.device_ms);
  }
  return best;
}

}  // namespace

extern "C" {

vp_status vp_autotune(void* p, const vp_autotune_opts* o, vp_config* best_out, vp_tune_report* rep) {
  if (!p) return VP_ERR_INVALID;
  vp_autotune_opts opt;
  memset(&opt, 0, sizeof(opt));
  if (o) opt = *o;
  const double budget_s = opt.time_budget_s > 0 ? opt.time_budget_s : 60.0;
  const int gran = opt.sm_granularity > 0 ? opt.sm_granularity : 4;
  const int max_cand = opt.max_candidates > 0 ? opt.max_candidates : 400;
  const int reps = opt.repeats > 0 ? opt.repeats : 1;
  const uint32_t allowed = opt.models_allowed ? opt.models_allowed : 0xFu;
  std::vector<int> divs;
  for (int i = 0; i < 4 && opt.batch_choices[i] > 0; ++i) divs.push_back(opt.batch_choices[i]);
  if (divs.empty()) divs.push_back(1);

  vp_tune_report R;
  memset(&R, 0, sizeof(R));
  // ---- profiling component (L13, L45): max resident blocks per SM of each stage kernel
  vp_status rc = vp_profile(p, R.max_blocks_per_sm, R.regs_per_thread, R.smem_per_block);
  if (rc != VP_OK) return rc;
  const int S = vpi_num_stages(p);
  const int N = vpi_num_sms(p);
  const double saved_timeout = vpi_timeout(p);
  const auto t0 = std::chrono::steady_clock::now();
  auto elapsed = [&] { return std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count(); };

  struct Cand {
    double ms;
    vp_config c;
  };
  std::vector<Cand> fastest;  // fastest candidates seen (single-run times are noisy)
  double mintime = 1e30;
  vp_config best;
  memset(&best, 0, sizeof(best));
  bool have_best = false;
  const bool debug = getenv("VP_TUNE_DEBUG") != nullptr;
  vp_status fatal = VP_OK;
  auto consider = [&](const vp_config& c, double limit) -> double {
    bool to = false;
    if (fatal != VP_OK) return -1.0;
    if (debug) {
      char buf[4096];
      vp_config_to_string(&c, buf, sizeof(buf));
      fprintf(stderr, "[vp_tune %.2fs] try limit=%.3fms %.160s\n", elapsed(), limit, buf);
      fflush(stderr);
    }
    double t = timeoutexec(p, c, limit, reps, &to, &fatal);
    if (debug) {
      fprintf(stderr, "[vp_tune %.2fs]   -> %.3f ms%s%s\n", elapsed(), t, to ? " (timeout)" : "",
              fatal != VP_OK ? " (CUDA error: search stopped)" : "");
      fflush(stderr);
    }
    R.candidates_run++;
    if (to) R.candidates_timed_out++;
    if (t > 0 && t < mintime) {
      mintime = t;
      best = c;
      have_best = true;
    }
    if (t > 0) {  // keep the fastest few for the final re-timing
      fastest.push_back({t, c});
      std::sort(fastest.begin(), fastest.end(), [](const Cand& a, const Cand& b) { return a.ms < b.ms; });
      if (fastest.size() > 4) fastest.pop_back();
    }
    return t;
  };

  // ---- baselines (KBK, megakernel); the megakernel run also profiles per-stage work
  double work[VP_MAX_STAGES] = {};
  {
    vp_config c;
    memset(&c, 0, sizeof(c));
    c.model = VP_KBK;
    R.baseline_kbk_ms = consider(c, saved_timeout);
    c.model = VP_MEGAKERNEL;
    uint32_t old = vpi_swap_flags(p, VP_FLAG_TIMERS);
    vp_run_stats st;
    if (vp_configure_config(p, &c) == VP_OK) {
      vp_set_timeout(p, saved_timeout);
      if (vp_run(p, nullptr, &st) == VP_OK && vp_run(p, nullptr, &st) == VP_OK)
        for (int s = 0; s < S; ++s) work[s] = (double)st.stage_exec_ns[s] + (double)st.stage_flush_ns[s];
    }
    vpi_swap_flags(p, old);
    R.baseline_mega_ms = consider(c, have_best ? 4.0 * mintime : saved_timeout);
  }
  double wsum = 0;
  for (int s = 0; s < S; ++s) wsum += work[s];
  if (wsum <= 0) {
    wsum = 0;
    for (int s = 0; s < S; ++s) work[s] = 1.0, wsum += 1.0;
  }
  auto seed_split = [&](Shape& sh) {
    if (sh.G == 1) {
      sh.sms[0] = N;
      return;
    }
    int used = 0;
    for (int g = 0; g < sh.G; ++g) {
      double gw = 0;
      for (int s = sh.lo[g]; s <= sh.hi[g]; ++s) gw += work[s];
      sh.sms[g] = std::max(gran, (int)(N * gw / wsum / gran + 0.5) * gran);
      used += sh.sms[g];
    }
    // fix the total to N: shrink / grow the largest group
    int big = 0;
    for (int g = 1; g < sh.G; ++g)
      if (sh.sms[g] > sh.sms[big]) big = g;
    sh.sms[big] += N - used;
    if (sh.sms[big] < gran) sh.sms[big] = gran;
  };

  // ---- phase 1: every grouping x model assignment, work-proportional SM split
  std::vector<Shape> shapes;
  for (int gmask = 0; gmask < (1 << (S - 1)); ++gmask) {
    Shape sh;
    memset(&sh, 0, sizeof(sh));
    sh.div = 1;
    sh.lo[0] = 0;
    for (int s = 0; s < S; ++s)
      if (s == S - 1 || ((gmask >> s) & 1)) {
        sh.hi[sh.G++] = s;
        if (s + 1 < S) sh.lo[sh.G] = s + 1;
      }
    std::vector<std::vector<int>> choices(sh.G);
    for (int g = 0; g < sh.G; ++g) {
      const bool multi = sh.hi[g] > sh.lo[g];
      if ((allowed >> VP_GROUP_MEGA) & 1) choices[g].push_back(VP_GROUP_MEGA);
      if (((allowed >> VP_GROUP_RTC) & 1) && multi && vpi_rtc_legal(p, sh.lo[g], sh.hi[g])) choices[g].push_back(VP_GROUP_RTC);
      if (((allowed >> VP_GROUP_FINE) & 1) && multi) choices[g].push_back(VP_GROUP_FINE);
      if ((allowed >> VP_GROUP_KBK) & 1) choices[g].push_back(VP_GROUP_KBK);
      if (choices[g].empty()) choices[g].push_back(VP_GROUP_MEGA);
    }
    std::vector<int> idx(sh.G, 0);
    for (;;) {
      bool all_kbk = true;
      for (int g = 0; g < sh.G; ++g) {
        sh.gm[g] = choices[g][idx[g]];
        all_kbk &= sh.gm[g] == VP_GROUP_KBK;
      }
      if (!all_kbk && !(sh.G == 1 && sh.gm[0] == VP_GROUP_MEGA)) {  // those are the baselines
        seed_split(sh);
        shapes.push_back(sh);
      }
      int g = 0;
      while (g < sh.G && ++idx[g] == (int)choices[g].size()) idx[g++] = 0;
      if (g == sh.G) break;
    }
  }
  R.candidates_total = (int)shapes.size() + 2;
  // Phase 1 runs with a lenient limit (2x the best so far): a shape whose seed split is
  // off still gets a time, so it can be ranked and refined in phase 2.
  std::vector<std::pair<double, Shape>> scored;
  for (const Shape& sh : shapes) {
    if (elapsed() > budget_s || R.candidates_run >= max_cand) break;
    double t = consider(to_config(p, S, sh), 2.0 * mintime);
    if (t > 0) scored.push_back({t, sh});
  }
  if (((allowed >> VP_GROUP_RTC) & 1) && vpi_rtc_legal(p, 0, S - 1) && elapsed() < budget_s) {
    vp_config c;
    memset(&c, 0, sizeof(c));
    c.model = VP_RTC;
    consider(c, mintime);
    R.candidates_total++;
  }

  // ---- phase 2: SM-split and batch refinement around the best phase-1 shapes
  std::sort(scored.begin(), scored.end(), [](const auto& a, const auto& b) { return a.first < b.first; });
  const int top = std::min<int>(4, (int)scored.size());
  for (int k = 0; k < top; ++k) {
    Shape base = scored[k].second;
    std::vector<Shape> nb;
    if (base.G == 2) {
      for (int a = gran; a <= N - gran; a += gran)
        if (a != base.sms[0]) {
          Shape v = base;
          v.sms[0] = a;
          v.sms[1] = N - a;
          nb.push_back(v);
        }
    } else if (base.G > 2) {
      for (int i = 0; i < base.G; ++i)
        for (int j = 0; j < base.G; ++j)
          if (i != j)
            for (int d : {1, 2, 4, 8}) {
              Shape v = base;
              v.sms[i] -= d * gran;
              v.sms[j] += d * gran;
              if (v.sms[i] >= gran) nb.push_back(v);
            }
    }
    // order the split neighbours by distance from the seed (closest first)
    std::sort(nb.begin(), nb.end(), [&](const Shape& x, const Shape& y) {
      return std::abs(x.sms[0] - base.sms[0]) < std::abs(y.sms[0] - base.sms[0]);
    });
    for (int d : divs)
      if (d != 1) {
        Shape v = base;
        v.div = d;
        nb.insert(nb.begin(), v);
      }
    R.candidates_total += (int)nb.size();
    for (const Shape& v : nb) {
      if (elapsed() > budget_s || R.candidates_run >= max_cand) break;
      consider(to_config(p, S, v), mintime);
    }
  }

  // Final re-timing: the fastest few candidates (the baselines included) run again
  // with more repeats; the search's single-run times decide only which ones get here.
  if (fatal == VP_OK && fastest.size() > 1) {
    double best_ms = 1e30;
    for (const Cand& k : fastest) {
      bool to = false;
      const double t = timeoutexec(p, k.c, 2.0 * k.ms, std::max(3, reps), &to, &fatal);  // (not a new candidate)
      if (fatal != VP_OK) break;
      if (t > 0 && t < best_ms) {
        best_ms = t;
        best = k.c;
      }
    }
    if (best_ms < 1e30) mintime = best_ms;
  }
  vp_set_timeout(p, saved_timeout);
  if (fatal != VP_OK) return fatal;  // vp_last_error holds the CUDA message
  if (!have_best) {
    vpi_set_error(p, "autotune: no candidate ran successfully");
    return VP_ERR_CUDA;
  }
  rc = vp_configure_config(p, &best);
  if (rc != VP_OK) return rc;
  R.best_ms = mintime;
  if (best_out) *best_out = best;
  if (rep) *rep = R;
  return VP_OK;
}

// Text form: "vpcfg1 model=M batch=B binding=0|1 groups=G gos=a,b,.. gm=.. bps=.. bat=.. mask0=hex.hex.. ..."
vp_status vp_config_to_string(const vp_config* c, char* buf, size_t len) {
  if (!c || !buf || len == 0) return VP_ERR_INVALID;
  std::string s = "vpcfg1 model=" + std::to_string(c->model) + " batch=" + std::to_string(c->batch) +
                  " binding=" + std::to_string(c->has_binding);
  if (c->has_binding) {
    const vp_sm_binding& b = c->binding;
    s += " groups=" + std::to_string(b.num_groups);
    auto arr = [&](const char* name, const int* v) {
      s += std::string(" ") + name + "=";
      for (int i = 0; i < VP_MAX_STAGES; ++i) s += std::to_string(v[i]) + (i + 1 < VP_MAX_STAGES ? "," : "");
    };
    arr("gos", b.group_of_stage);
    arr("gm", b.group_model);
    arr("bps", b.blocks_per_sm);
    arr("bat", b.batch);
    for (int g = 0; g < VP_MAX_STAGES; ++g) {
      char tmp[16];
      s += " mask" + std::to_string(g) + "=";
      for (int w = 0; w < VP_MAX_SM / 32; ++w) {
        snprintf(tmp, sizeof(tmp), "%08x", b.group_sm_mask[g][w]);
        s += tmp;
        if (w + 1 < VP_MAX_SM / 32) s += ".";
      }
    }
  }
  if (s.size() + 1 > len) return VP_ERR_INVALID;
  memcpy(buf, s.c_str(), s.size() + 1);
  return VP_OK;
}

vp_status vp_config_from_string(const char* str, vp_config* out) {
  if (!str || !out) return VP_ERR_INVALID;
  vp_config c;
  memset(&c, 0, sizeof(c));
  if (strncmp(str, "vpcfg1 ", 7) != 0) return VP_ERR_INVALID;
  std::string s(str + 7);
  size_t pos = 0;
  auto ints = [](const std::string& v, int* dst) {
    int i = 0;
    size_t a = 0;
    while (i < VP_MAX_STAGES && a <= v.size()) {
      size_t b = v.find(',', a);
      dst[i++] = atoi(v.substr(a, b == std::string::npos ? std::string::npos : b - a).c_str());
      if (b == std::string::npos) break;
      a = b + 1;
    }
  };
  while (pos < s.size()) {
    size_t sp = s.find(' ', pos);
    std::string tok = s.substr(pos, sp == std::string::npos ? std::string::npos : sp - pos);
    pos = sp == std::string::npos ? s.size() : sp + 1;
    size_t eq = tok.find('=');
    if (eq == std::string::npos) continue;
    std::string k = tok.substr(0, eq), v = tok.substr(eq + 1);
    if (k == "model") c.model = atoi(v.c_str());
    else if (k == "batch") c.batch = atoi(v.c_str());
    else if (k == "binding") c.has_binding = atoi(v.c_str());
    else if (k == "groups") c.binding.num_groups = atoi(v.c_str());
    else if (k == "gos") ints(v, c.binding.group_of_stage);
    else if (k == "gm") ints(v, c.binding.group_model);
    else if (k == "bps") ints(v, c.binding.blocks_per_sm);
    else if (k == "bat") ints(v, c.binding.batch);
    else if (k.rfind("mask", 0) == 0) {
      int g = atoi(k.c_str() + 4);
      if (g < 0 || g >= VP_MAX_STAGES) return VP_ERR_INVALID;
      size_t a = 0;
      for (int w = 0; w < VP_MAX_SM / 32 && a < v.size(); ++w) {
        c.binding.group_sm_mask[g][w] = (uint32_t)strtoul(v.substr(a, 8).c_str(), nullptr, 16);
        a += 9;
      }
    } else {
      return VP_ERR_INVALID;
    }
  }
  if (c.model < VP_RTC || c.model > VP_KBK_GRAPH) return VP_ERR_INVALID;
  *out = c;
  return VP_OK;
}

}  // extern "C"
