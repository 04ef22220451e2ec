// Diagnostics: print the evaluation-kernel source codegen.cpp emits for one kernel and
// variant (no GPU, no NVRTC), e.g. to check a multi-seed variant with nvcc -Xptxas -v.
//   g++ -std=c++17 -I paper_conf_ipps_lig12_b200/csrc tools/gen_variant.cpp \
//       paper_conf_ipps_lig12_b200/csrc/front.cpp paper_conf_ipps_lig12_b200/csrc/codegen.cpp -o /tmp/gv/gen
//   /tmp/gv/gen subjects/reduce1.pgk FAST MS CHECKS
#include <cstdio>
#include <cstdlib>
#include <fstream>
#include <sstream>

#include "front.hpp"

int main(int argc, char** argv) {
    if (argc < 2) return 2;
    std::ifstream f(argv[1]);
    std::stringstream ss;
    ss << f.rdbuf();
    auto K = pgf::parse_kernel(ss.str());
    pgf::CodegenOptions o;
    o.fast = argc > 2 && std::atoi(argv[2]);
    o.ms = argc > 3 ? (uint32_t)std::atoi(argv[3]) : 1u;
    o.checks = argc > 4 ? (uint32_t)std::atoi(argv[4]) : 6u;
    std::fprintf(stderr, "seed_oblivious: %d\n", (int)pgf::seed_oblivious(*K));
    std::fputs(pgf::generate_cuda(*K, o).c_str(), stdout);
    return 0;
}
