// sf_internal.h — internal model of the stencil-DAG executor (host side).
//
// Program model: kernels, arrays, statements and their dependency edges are the
// paper's DDG/OEG (§2, §3.2.3).  A Launch is one generated
// kernel: a fused group of the plan ("new kernel") or one
// original kernel in unfused mode ("no fusion", §5.5.1).
#pragma once

#include <cstdint>
#include <array>
#include <map>
#include <memory>
#include <mutex>
#include <set>
#include <string>
#include <vector>

#include "stencilfuse.h"

namespace sf {

struct Tap { int arr, dx, dy, dz; };
struct Term { double coef; Tap a; bool has_b; Tap b; };
struct Stmt {
    int kernel, local, gid;  // kernel index, index inside kernel, global program-order id
    int out;
    std::vector<Term> terms;
    int64_t box[6] = {0, 0, 0, 0, 0, 0};  // loop bounds, global interior coordinates (R2')
    bool boxed = false;                   // box is smaller than the whole interior
};
struct Kernel { std::string name; std::vector<int> stmts; };
struct ArrayDesc { std::string name; sp_role role; };

struct Options {
    int fmad = 1;
    int tile_x = 0, tile_y = 0, zchunk = 0, threads = 0, prefetch = -1;
    int loader = 0;  // 0: TMA + mbarrier ring, 1: cooperative ld.global -> st.shared
    int block_x = 0, block_y = 0, block_cby = 0;  // register-block overrides (0 = chooser)
    int zqueue = 0;  // z-queues cost registers/occupancy more than they save (measured r1)
    int suspend_hint = 0;  // ns hint of mbarrier.try_wait (0 = none)
    int l2pf = 1;          // TMA L2 prefetch distance in steps beyond the ring (0 = off;
                           // r1s3: 1 wins with the prefetch-1 rings: C2 -3.4 %, C5 -2 %, C4 -0.7 %)
    int coef_const = 0;    // fp64: 1 = __constant__ table (r1: 35 % slower, hoisted), 2 = table read
                           // per use through a per-step zero (one LDCU.64 per coefficient)
    int pdl = 1;        // programmatic dependent launch: 1 = fused groups, 2 = all, 0 = off
    int acc_split = 1;  // >1: interleaved partial sums in the perf build (no gain measured r1)
    int factor = 1;     // perf build: terms sharing one b operand are summed, then multiplied once
    int zwave = 0;          // z-wave schedule: planes per wave (0 = one launch per group per step)
    int zwave_streams = 2;  // waves in flight (streams) of the z-wave schedule
    int xpush = 0;  // several ranks: stores push in-step halo planes into the neighbours' ghosts
    int fastpath = 0;  // emit a second, predicate-free step body for interior tiles / planes
                       // (r2: 40 % fewer issued instructions per step, but the doubled code
                       // overflows the 32 KB instruction cache: C4 +2 %, C2 +12 % slower)
    int minblocks = 1; // __launch_bounds__ minimum resident CTAs (register budget for ptxas)
    int cluster_x = 1; // > 1: CTAs per cluster along x sharing x-halos of smem stages over DSMEM
    int frame = 0;     // region-vector evaluation of fused launches (see stencilfuse.h "frame")
    int rename = 1;    // fused mode, one rank: every later writer group of a TEMP gets its own
                       // buffer instance (no WAR/WAW through TEMP reuse between groups)
    int streams = 2;   // fused mode, one rank: launches on up to this many streams along the
                       // group dependency DAG (events between streams); r2: C4 -8.3 %
    int dagsched = 0;  // DAG stream assignment: 0 follow the latest dependency, 1 roots on their own stream
    int dagprio = 0;   // launch-DAG streams' priority: 0 default, 1 higher, 2 lower than default
    int pbar = 0;      // 1: "slot free" via named barriers (producer blocks in bar.sync, no polling)
    int pow2ring = 0;  // ring depths rounded up to powers of two (slot = mask, more shared memory)
    int phint = 0;     // > 0: producer waits with try_wait suspend-time hint (ns) instead of psleep
    int psleep = 32;   // producer waits for a free ring slot with nanosleep back-off (ns; 0 = spin):
                       // r2: the spinning producer warp issued 28 % of sf_fused_5's instructions;
                       // 32 ns back-off: C4 -3.6 %, C3 -1.2 %, C2 -0.7 % (interleaved A/B)
    int halo_sel = 0;  // halo points: expression always evaluated, ghost value selected after
                       // (no branch around the loads: several halo points' loads interleave)
    int regcap = 1; // recompile a few registers tighter when that adds a resident CTA:
                    // 0 never, 1 peer-push kernels, 2 every kernel
};

// ---------------------------------------------------------------- analysis
enum class Keep { Dead, Reg, Smem };

// A term operand after resolution inside a launch: an on-chip stage (position
// in the launch) or an external input (index into Launch::in).
struct Src { bool stage; int idx; int dx, dy, dz; };
struct TermR { double coef; Src a; bool has_b; Src b; };

struct Stage {
    int gid = -1;           // statement
    int out = -1;           // array written
    std::vector<TermR> terms;
    bool stored = false;    // written back to HBM (live-out, reading R6)
    bool needed = false;    // computed at all
    // computed region relative to the tile: x in [-ex0, TX+ex1), y in [-ey0, TY+ey1)
    int ex0 = 0, ex1 = 0, ey0 = 0, ey1 = 0;
    // computed planes [loff, zc-1+lead] relative to the chunk; computed at step k: plane k+lead
    int loff = 0, lead = 0;
    int depth = 1;          // planes kept on chip (ring / queue)
    Keep keep = Keep::Dead;
    int cls = -1;           // region class (thread->point mapping)
    bool war_barrier = false;  // needs a CTA barrier before its store (R11 exception)
    int sx0 = 0;            // smem layout left extension, ex0 rounded up to 16 B (vector alignment)
};

struct Input {
    int arr = -1;
    int ex0 = 0, ex1 = 0, ey0 = 0, ey1 = 0;  // region relative to the tile
    int alo = 0, ahi = 0;   // planes read at step k: [k+alo, k+ahi]
    int qlo = 0;            // first plane needed (relative to chunk); last = zc-1+ahi
    int bx0 = 0;            // box x extension, ex0 rounded up to 16 B (TMA box start alignment)
};

struct RegionClass { int x0, x1, y0, y1; };  // relative to the tile, half-open

struct Launch {
    std::string name;
    std::vector<int> members;  // statement gids, program order
    std::vector<Stage> st;
    std::vector<Input> in;
    std::vector<RegionClass> cls;
    std::vector<int> arr_slot;   // array id -> pointer slot in params (-1 unused)
    std::vector<int> slot_arr;   // pointer slot -> array id
    int kfirst = 0;              // first step (<= 0), relative to the chunk
    int z_below = 0, z_above = 0;
    // configuration
    int tx = 0, ty = 0, zc = 0, nt = 0, pf = 0;
    int nth = 0;                 // threads per CTA (compute threads nt + producer warp)
    int vx = 1, vy = 1, cby = 1; // register block of a thread: cby blocks of vx x vy core points
    int zq = 0;                  // z-queues for values read at several planes
    int est_regs = 0;            // register estimate used by the tile chooser
    double t_model = 0;          // modelled launch time (s)
    int ntx = 0, nty = 0, nch = 0;
    int64_t smem = 0;
    int rw_pad = 2;              // input row padding granularity (elements)
    // layout of smem (bytes) per input ring / stage ring
    std::vector<int64_t> in_off, in_plane;   // plane size in elements (padded)
    std::vector<int> in_rw, in_rh, in_depth;  // ring depth (planes)
    std::vector<int64_t> st_off, st_plane;
    std::vector<int> st_w, st_h, st_depth;
    int64_t bar_off = 0;
    int n_bars = 0;
    int64_t ready_off = 0;       // cluster "plane ready" mbarriers (one per shared-memory stage)
    int cx = 1;                  // CTAs per cluster along x (1: no cluster)
    int nbar_full = 1, nbar_empty = 1;  // per-step batch barriers (powers of two)
    // report
    double bytes_alg = 0, flops_alg = 0, bytes_exec = 0, flops_exec = 0, smem_pt = 0;
    // jit
    std::string fn;
    std::string nvtx;            // NVTX range name of a launch: "<fn> <group name>"
    std::string source;
    std::string cubin;
    int regs = -1;
    void *func = nullptr;    // CUfunction
    void *module = nullptr;  // CUmodule
    size_t param_size = 0, ptr_off = 0, int_off = 0;
    // peer-push halo exchange (option xpush, several ranks): stage `stage` also stores
    // its bottom `dn` planes into the lower neighbour's top ghost and its top `up`
    // planes into the upper neighbour's bottom ghost
    struct Push { int stage, dn, up; };
    std::vector<Push> pushes;
    bool xp = false;         // kernel carries the peer-push signal protocol
    int xp_dw = 0;           // chunks within xp_dw planes of a slab end wait for the neighbours
    size_t xp_off = 0;       // param offset of the peer-push section
    bool dead = false;       // nothing to compute (all stages dead)
    bool pdl = false;        // launched with programmatic stream serialization
    int fastpath = -1;       // per-launch pin of the "fastpath" codegen variant (-1: option)
    int frame_pin = -1;      // per-launch pin of the "frame" evaluation mode (-1: option)
    bool fr = false;         // region-vector evaluation (resolved from pin/option/eligibility)
    bool fr2 = false;        // frame mode with position-stable units and register z-reuse
    bool pbar = false;       // "slot free" signalled through named barriers (codegen)
};

struct Mode {
    std::vector<Launch> launches;
    bool analyzed = false;
    bool compiled = false;
    bool loaded = false;
    uint64_t maps_version = ~0ull;
    struct alignas(64) Blk { unsigned char b[64]; };
    std::vector<std::vector<Blk>> params;  // per launch: tensor maps + pointers + ints
    std::vector<int> wave_off;  // z-wave schedule: plane offset (skew) per launch
    // multi-rank halo exchange schedule: per launch, the ghost planes to receive first
    struct Xfer { int arr, below, above; };
    std::vector<std::vector<Xfer>> xsched;
    bool xsched_ok = false;
    // TEMP renaming and the launch DAG (options rename / streams, one rank, fused mode):
    // per launch and array the buffer instance its HBM reads / stores use (0 = the bound
    // buffer, k > 0 = the program's k-th shadow of that array), the launches each depends
    // on (RAW/WAR/WAW on instances) and the stream index each is issued on
    std::vector<std::vector<int>> rd_inst, wr_inst;
    std::vector<int> n_inst;
    std::vector<std::vector<int>> deps;
    std::vector<int> stream_of;
    bool dag_ok = false;
    std::vector<void *> shadow_src;  // per array: the bound buffer its shadows were copied from
};

}  // namespace sf

namespace sf { struct LoopHub; }
struct sp_comm_s {
    void *nccl = nullptr;  // ncclComm_t (null for a loopback communicator)
    int nranks = 1, rank = 0, device = 0;
    void *comm_stream = nullptr;  // cudaStream_t used for exchanges
    std::shared_ptr<sf::LoopHub> hub;  // in-process virtual ranks (test transport)
};

struct stencil_program_s {
    sp_grid grid{};
    int elem = 8;
    std::vector<sf::ArrayDesc> arrays;
    std::vector<sf::Kernel> kernels;
    std::vector<sf::Stmt> stmts;
    std::vector<sp_edge> edges;
    sp_layout layout{};
    int64_t plane = 0;           // x_pitch * y_alloc
    int64_t zint_lo = 0, zint_hi = 0;  // global interior in local z coordinates
    std::vector<void *> ptrs;
    uint64_t bind_version = 0;
    sp_comm *comm = nullptr;
    sf::Options opt;
    sf::Mode unfused, fused;
    bool has_plan = false;
    std::vector<std::vector<int>> plan_groups;  // gids per group
    int num_sms = 148;
    std::vector<void *> events;  // cudaEvent_t pool for exchange overlap
    bool no_pdl = false;         // multi-rank schedule: plain stream order between launches
    std::vector<void *> wave_streams, wave_events;  // z-wave schedule: streams, events
    std::vector<void *> dag_streams, dag_events;    // launch-DAG streams (option streams)
    std::vector<std::vector<void *>> shadow;        // per array: renamed TEMP instances (option rename)
    std::map<int, sp_tile_config> tune_fused, tune_unfused;  // sp_plan_tune overrides
    // peer-push exchange: neighbours' buffers of each array (0 = below, 1 = above),
    // this program's signal block (u64 from_dn, from_up, self; u32 cta counter) and
    // the neighbours' signal blocks, all mapped in this process
    std::vector<std::array<void *, 2>> peer;
    void *sig = nullptr;
    void *peer_sig[2] = {nullptr, nullptr};
};

namespace sf {
// errors --------------------------------------------------------------------
void set_error(const std::string &msg);
struct Error { sp_status code; std::string msg; };
[[noreturn]] void fail(sp_status code, const std::string &msg);

// program.cpp
void build_edges(stencil_program *p);
std::vector<int> fission_components(const stencil_program *p, int kernel, int *n_comp);

// plan.cpp
void analyze_mode(stencil_program *p, bool fused, const std::vector<std::vector<int>> &groups,
                  Mode &out);
void fill_report(const stencil_program *p, const Launch &L, sp_group_report *r);
std::vector<std::vector<int>> greedy_plan(stencil_program *p);
Launch analyze_group(const stencil_program *p, const std::vector<int> &members,
                     const std::set<int> &stored_gids);
void choose_config(const stencil_program *p, Launch &L, bool quick = false);
void model(const stencil_program *p, Launch &L);
void live_out(const stencil_program *p, bool fused, const std::vector<std::vector<int>> &groups,
              std::vector<std::set<int>> &stored);
std::vector<std::vector<int>> fission_units(const stencil_program *p);

// search.cpp: lazy-fission plan search (NEXT #1)
std::vector<std::vector<int>> search_plan(stencil_program *p, const sp_search_options &o, void *stream,
                                          sp_search_report *rep, std::vector<sp_tile_config> *configs);

// codegen.cpp
std::string generate_launch(const stencil_program *p, Launch &L, int index, bool fused);
void core_geometry(const Launch &L, int *xt, int *yt);
int codegen_regs(const stencil_program *p, const Launch &L);
double codegen_smem_loads(const Launch &L);  // shared-memory loads per core point (all stages)

// jit.cpp
void compile_mode(stencil_program *p, Mode &m);
void load_mode(stencil_program *p, Mode &m);
// TEMP instances and the launch DAG of a mode (options rename / streams); idempotent
void dag_analysis(stencil_program *p, Mode &m, bool fused);
// shadow buffers of renamed TEMPs: allocated and initialised from the bound buffer (ghost
// cells) when the bindings changed, on `stream`
void prepare_shadows(stencil_program *p, Mode &m, void *stream);
// one launch over output planes [z0, z1) and [z2, z3) of the slab (z1 < 0: the
// whole slab; an empty second range by default), each tiled by chunks of zc planes
void launch(stencil_program *p, Mode &m, int i, void *stream, int z0 = 0, int z1 = -1, int z2 = 0,
            int z3 = 0);
void ensure_cuda();
void *signal_block(stencil_program *p);  // allocated (zeroed) on first use
bool driver_mem_range(unsigned long long *base, size_t *size, unsigned long long p);  // cuMemGetAddressRange
void unload_mode(Mode &m);

// comm.cpp
// receive `below` planes into the bottom ghost and `above` planes into the top
// ghost of each array (the neighbours send the matching interior planes)
void exchange(stencil_program *p, const std::vector<Mode::Xfer> &x, void *stream);
void exchange_schedule(const stencil_program *p, Mode &m);
void *comm_stream(sp_comm *c);  // the communicator's exchange stream (created on first use)
}  // namespace sf
