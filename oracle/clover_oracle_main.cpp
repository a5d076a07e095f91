/*
 * clover_oracle_main.cpp -- command-line driver of the CPU ORACLE
 * (SURVEY.md 8(c) c.15 "Oracle I/O contract").
 *
 * TEST INFRASTRUCTURE ONLY, like the library it links (clover_oracle.cpp):
 * tests/ and the bench's reference leg may run it; the product path never
 * does.  It shares no code with paper_conf_cluster_regulymg15_b200/.
 *
 *   clover_oracle [--steps N] [--summary-every K] [--dump DIR] DECK
 *
 * DECK is a CloverLeaf-style text deck (the reference's clover.in form,
 * SURVEY 8(c) c.15):
 *
 *   *clover
 *    state 1 density=0.2 energy=1.0
 *    state 2 density=1.0 energy=2.5 geometry=rectangle xmin=0.0 xmax=5.0 ymin=0.0 ymax=2.0
 *    x_cells=64  y_cells=64  xmin=0.0 ymin=0.0 xmax=10.0 ymax=10.0
 *    initial_timestep=0.04  max_timestep=0.04  timestep_rise=1.5  end_step=20
 *   *endclover
 *
 * plus the test keys advect_x_first=0|1, face_mirror=geometric|cellcentre
 * (reading A7), summary_every=K, dtmin / dtc_safe / dtu_safe / dtv_safe /
 * dtdiv_safe.  Lines outside *clover ... *endclover and text after '!' are
 * ignored.  (JSON decks are converted to this form by oracle/deck.py.)
 *
 * Output (stdout, JSON lines; every double printed with %.17g, round-trip
 * exact): one {"step","time","dt"} line per step, and a summary line
 * {"summary": step, "vol", "mass", "ie", "ke", "press", "density",
 * "pressure", "total"} at step 0, every K steps and after the last step
 * (c.12 field_summary; density = mass/vol, pressure = press/vol,
 * total = ie+ke, as the reference prints them).
 * --dump DIR writes the global interior of every field after the last step
 * as raw little-endian fp64, row-major, j fastest (cells nx*ny, nodes
 * (nx+1)*(ny+1), x-faces (nx+1)*ny, y-faces nx*(ny+1)) into DIR/<field>.f64:
 * the clover_read_field convention, so GPU parity is a byte compare.
 * Exit status 0; 2 on a bad deck; 5 on dt < dtmin (the step log so far is
 * printed).
 */
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <sstream>
#include <string>
#include <vector>

#include "clover_oracle.h"

namespace {

struct Deck {
  oracle_grid g{};
  std::vector<oracle_state> states;
  int end_step = 0;
  int summary_every = 0;
  bool ok = true;
  std::string err;
};

bool parse_double(const std::string& v, double* out) {
  char* end = nullptr;
  *out = std::strtod(v.c_str(), &end);
  return end && *end == '\0' && !v.empty();
}

/* the reference's input is Fortran-ish: keys are case-insensitive */
std::string lower(std::string s) {
  for (auto& ch : s) ch = (char)std::tolower((unsigned char)ch);
  return s;
}

Deck parse_deck(std::istream& in) {
  Deck d;
  d.g.xmin = 0.0; d.g.ymin = 0.0; d.g.xmax = 100.0; d.g.ymax = 100.0;  // reference defaults
  d.g.x_cells = 10; d.g.y_cells = 10;
  d.g.dtinit = 0.1; d.g.dtmax = 1.0; d.g.dtrise = 1.5;
  d.g.advect_x_first = 1;
  d.g.face_mirror = OR_MIRROR_GEOMETRIC;
  bool inside = false, seen = false;
  std::string line;
  auto fail = [&](const std::string& m) { d.ok = false; if (d.err.empty()) d.err = m; };
  while (std::getline(in, line)) {
    const size_t bang = line.find('!');
    if (bang != std::string::npos) line.resize(bang);
    std::istringstream ls(line);
    std::vector<std::string> tok;
    for (std::string t; ls >> t;) tok.push_back(t);
    if (tok.empty()) continue;
    const std::string t0 = lower(tok[0]);
    if (t0 == "*clover") { inside = true; seen = true; continue; }
    if (t0 == "*endclover") { inside = false; continue; }
    if (!inside) continue;
    size_t i = 0;
    oracle_state* st = nullptr;
    if (t0 == "state") {
      if (tok.size() < 2) { fail("state without a number"); continue; }
      const int n = std::atoi(tok[1].c_str());
      if (n < 1) { fail("state numbers start at 1"); continue; }
      if ((int)d.states.size() < n) d.states.resize(n, oracle_state{});
      st = &d.states[n - 1];
      if (st->geometry == 0) st->geometry = OR_GEOM_RECT;
      i = 2;
    }
    for (; i < tok.size(); ++i) {
      const size_t eq = tok[i].find('=');
      if (eq == std::string::npos) { fail("expected key=value: " + tok[i]); continue; }
      const std::string k = lower(tok[i].substr(0, eq)), v = tok[i].substr(eq + 1);
      double x = 0.0;
      if (st) {
        if (k == "geometry") {
          const std::string g = lower(v);
          st->geometry = g == "rectangle" ? OR_GEOM_RECT : g == "circle" ? OR_GEOM_CIRCLE
                       : g == "point" ? OR_GEOM_POINT : 0;
          if (!st->geometry) fail("unknown geometry " + v);
          continue;
        }
        if (!parse_double(v, &x)) { fail("bad number " + tok[i]); continue; }
        if (k == "density") st->density = x;
        else if (k == "energy") st->energy = x;
        else if (k == "xvel") st->xvel = x;
        else if (k == "yvel") st->yvel = x;
        else if (k == "xmin") st->xmin = x;
        else if (k == "xmax") st->xmax = x;
        else if (k == "ymin") st->ymin = x;
        else if (k == "ymax") st->ymax = x;
        else if (k == "radius") st->radius = x;
        else fail("unknown state key " + k);
        continue;
      }
      if (k == "face_mirror") {
        const std::string m = lower(v);
        if (m == "geometric" || m == "0") d.g.face_mirror = OR_MIRROR_GEOMETRIC;
        else if (m == "cellcentre" || m == "1") d.g.face_mirror = OR_MIRROR_CELLCENTRE;
        else fail("face_mirror must be geometric or cellcentre");
        continue;
      }
      if (!parse_double(v, &x)) { fail("bad number " + tok[i]); continue; }
      if (k == "x_cells") d.g.x_cells = (int32_t)x;
      else if (k == "y_cells") d.g.y_cells = (int32_t)x;
      else if (k == "xmin") d.g.xmin = x;
      else if (k == "ymin") d.g.ymin = x;
      else if (k == "xmax") d.g.xmax = x;
      else if (k == "ymax") d.g.ymax = x;
      else if (k == "initial_timestep") d.g.dtinit = x;
      else if (k == "max_timestep") d.g.dtmax = x;
      else if (k == "timestep_rise") d.g.dtrise = x;
      else if (k == "dtmin") d.g.dtmin = x;
      else if (k == "dtc_safe") d.g.dtc_safe = x;
      else if (k == "dtu_safe") d.g.dtu_safe = x;
      else if (k == "dtv_safe") d.g.dtv_safe = x;
      else if (k == "dtdiv_safe") d.g.dtdiv_safe = x;
      else if (k == "end_step") d.end_step = (int)x;
      else if (k == "advect_x_first") d.g.advect_x_first = (int32_t)x;
      else if (k == "summary_every" || k == "summary_frequency") d.summary_every = (int)x;
      else if (k == "test_problem" || k == "end_time" || k == "visit_frequency" ||
               k == "profiler_on")
        ;  // accepted, no effect here
      else fail("unknown key " + k);
    }
  }
  if (!seen) fail("no *clover block");
  if (d.states.empty()) fail("no states");
  for (auto& s : d.states)
    if (s.geometry == 0) s.geometry = OR_GEOM_RECT;
  return d;
}

void print_summary(oracle_ctx* c, int step) {
  double s[5];
  oracle_field_summary(c, s);
  std::printf("{\"summary\": %d, \"vol\": %.17g, \"mass\": %.17g, \"ie\": %.17g, \"ke\": %.17g, "
              "\"press\": %.17g, \"density\": %.17g, \"pressure\": %.17g, \"total\": %.17g}\n",
              step, s[0], s[1], s[2], s[3], s[4], s[1] / s[0], s[4] / s[0], s[2] + s[3]);
}

const struct { int id; const char* name; int ax, ay; } kFields[] = {
    {OF_DENSITY0, "density0", 0, 0},   {OF_ENERGY0, "energy0", 0, 0},
    {OF_PRESSURE, "pressure", 0, 0},   {OF_VISCOSITY, "viscosity", 0, 0},
    {OF_SOUNDSPEED, "soundspeed", 0, 0}, {OF_XVEL0, "xvel0", 1, 1},
    {OF_YVEL0, "yvel0", 1, 1},         {OF_VOL_FLUX_X, "vol_flux_x", 1, 0},
    {OF_VOL_FLUX_Y, "vol_flux_y", 0, 1}, {OF_MASS_FLUX_X, "mass_flux_x", 1, 0},
    {OF_MASS_FLUX_Y, "mass_flux_y", 0, 1}};

bool dump(oracle_ctx* c, const Deck& d, const std::string& dir) {
  for (const auto& f : kFields) {
    const int64_t n = (int64_t)(d.g.x_cells + f.ax) * (d.g.y_cells + f.ay);
    std::vector<double> buf((size_t)n);
    if (oracle_read_field(c, f.id, buf.data(), n) != 0) return false;
    const std::string path = dir + "/" + f.name + ".f64";
    FILE* fp = std::fopen(path.c_str(), "wb");
    if (!fp) return false;
    const size_t w = std::fwrite(buf.data(), sizeof(double), buf.size(), fp);
    std::fclose(fp);
    if (w != buf.size()) return false;
  }
  return true;
}

}  // namespace

int main(int argc, char** argv) {
  int steps = -1, every = -1;
  std::string dir, path;
  for (int a = 1; a < argc; ++a) {
    const std::string s = argv[a];
    if (s == "--steps" && a + 1 < argc) steps = std::atoi(argv[++a]);
    else if (s == "--summary-every" && a + 1 < argc) every = std::atoi(argv[++a]);
    else if (s == "--dump" && a + 1 < argc) dir = argv[++a];
    else if (!s.empty() && s[0] != '-') path = s;
    else {
      std::fprintf(stderr, "usage: clover_oracle [--steps N] [--summary-every K] [--dump DIR] DECK\n");
      return 2;
    }
  }
  std::ifstream in(path);
  if (!in) { std::fprintf(stderr, "cannot read deck %s\n", path.c_str()); return 2; }
  Deck d = parse_deck(in);
  if (!d.ok) { std::fprintf(stderr, "bad deck: %s\n", d.err.c_str()); return 2; }
  if (steps < 0) steps = d.end_step;
  if (every < 0) every = d.summary_every;
  oracle_ctx* c = oracle_create(&d.g, d.states.data(), (int32_t)d.states.size());
  if (!c) { std::fprintf(stderr, "the oracle rejected the deck\n"); return 2; }
  print_summary(c, 0);
  int rc = 0;
  for (int n = 1; n <= steps; ++n) {
    double dt = 0.0;
    if (oracle_step(c, 1, &dt) != 0) { rc = 5; break; }
    int32_t st; double t, dtl, dto;
    oracle_clock(c, &st, &t, &dtl, &dto);
    std::printf("{\"step\": %d, \"time\": %.17g, \"dt\": %.17g}\n", st, t, dt);
    if ((every > 0 && n % every == 0) || n == steps) print_summary(c, n);
  }
  if (rc == 0 && !dir.empty() && !dump(c, d, dir)) {
    std::fprintf(stderr, "dump to %s failed\n", dir.c_str());
    rc = 2;
  }
  oracle_destroy(c);
  return rc;
}
