// libdfg runtime: meshes, plans, the three execution strategies, the device
// memory ledger and the halo exchange.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <map>
#include <algorithm>
#include <memory>
#include <string>
#include <vector>

#include "codegen.hpp"
#include "jit.hpp"
#include "lang.hpp"

namespace dfg {

struct Binding {
  void* ptr = nullptr;
  bool on_device = false;
};

struct MeshImpl {
  DType dt = DType::F32;
  // local cells (nx, ny, nzl) of a global NX x NY x NZ mesh at offsets (i0, j0, k0)
  int64_t nx = 0, ny = 0, nzl = 0, NZ = 0, k0 = 0;
  int64_t NX = 0, NY = 0, i0 = 0, j0 = 0;
  int ghost = 0;     // ghost planes in z (slabs, blocks)
  int gxy = 0;       // ghost columns / rows in x and y (VisIt blocks, caller-filled)
  int64_t pitch = 0; // input row pitch in elements (blocks; 0 = nx + 2*gxy)
  int64_t xoff = 0;  // column of the first owned cell in an input row (blocks; 0 = gxy)
  bool ghosts_supplied = false;  // blocks: the caller fills every ghost cell (no exchange)
  int device = 0;
  bool markstein_safe = true;        // spacing tables inside the exact-division range
  int div2_mask = 0;                 // bit a: every divisor of axis a passed verify_div2 (fp32) / certify_div2 (fp64)
  std::vector<char> host_tab[3];     // per axis over the GLOBAL mesh: d | r | -d | yl (T), reading R1
  void* dev_tab[3] = {nullptr, nullptr, nullptr};
  std::map<std::string, Binding> fields;
  // halo transport
  int rank = 0, nranks = 1;
  void* nccl = nullptr;              // ncclComm_t
  std::weak_ptr<MeshImpl> link_lo, link_hi;
  // peer-memory halo (dfg_mesh_peer_export / dfg_mesh_link_peers): the fused
  // kernel reads the neighbours' boundary planes from their buffers (CUDA IPC
  // mappings; NVLink between GPUs); step flags order the accesses
  struct Peer {
    bool on = false;
    int64_t k0 = 0, nzl = 0, ghost = 0;
    std::map<std::string, void*> fields;  // mapped field bases (ghost plane 0 included)
    uint32_t* flags = nullptr;            // mapped flag words of the peer
  };
  Peer peer_lo, peer_hi;
  uint32_t* flags = nullptr;         // own flags: [0] ready, [16] lo done, [32] hi done (64-byte apart)
  uint32_t epoch = 0;                // executes of this mesh (every rank runs the same sequence)
  std::map<std::string, void*> exported;  // bindings at export time (must not change while linked)
  std::vector<void*> ipc_opened;     // cudaIpcOpenMemHandle bases to close
  ~MeshImpl();
  int64_t px() const { return pitch ? pitch : nx + 2 * gxy; }  // input row pitch
  int64_t gx() const { return xoff ? xoff : gxy; }   // first owned column of an input row
  int64_t py() const { return ny + 2 * gxy; }        // input rows per plane
  int64_t plane() const { return nx * ny; }          // owned cells per plane (output)
  int64_t in_plane() const { return px() * py(); }   // input plane incl. x/y ghosts
  int64_t cells() const { return nx * ny * nzl; }
  size_t field_bytes() const { return size_t(in_plane() * (nzl + 2 * ghost)) * dsize(dt); }
};

// The part of a mesh one fused launch covers: a whole mesh, a z-slab of a
// multi-GPU mesh, a VisIt-style block, or one z-chunk of the streamed
// strategy (ghost planes at local 0 and nzl+1 when ghost = 1; ghost columns /
// rows at local 0 and n+1 when gxy = 1).
struct SlabView {
  DType dt;
  int64_t nx, ny, nzl, NZ, k0;
  int ghost;
  int64_t NX, NY, i0, j0;
  int gxy;
  int64_t pitch, xoff;
  static SlabView of(const MeshImpl& m) {
    return SlabView{m.dt, m.nx, m.ny, m.nzl, m.NZ, m.k0, m.ghost, m.NX, m.NY, m.i0, m.j0, m.gxy, m.pitch, m.xoff};
  }
  int64_t px() const { return pitch ? pitch : nx + 2 * gxy; }
  int64_t gx() const { return xoff ? xoff : gxy; }
  int64_t py() const { return ny + 2 * gxy; }
};

constexpr int kStreamSlots = 3;  // ring depth of the streamed strategy

std::shared_ptr<MeshImpl> create_mesh(DType dt, int64_t nx, int64_t ny, int64_t nzl, const void* x, const void* y,
                                      const void* z, int64_t NZ, int64_t k0, int ghost);
// VisIt-style block (NEXT #4): local nx x ny x nz cells at (i0, j0, k0) of a
// global NX x NY x NZ mesh, global point coordinates, ghost = 0/1 cell shell
// on all six faces filled by the caller.
std::shared_ptr<MeshImpl> create_block(DType dt, int64_t nx, int64_t ny, int64_t nz, const void* x, const void* y,
                                       const void* z, int64_t NX, int64_t NY, int64_t NZ, int64_t i0, int64_t j0,
                                       int64_t k0, int ghost, int64_t pitch, int64_t xoff);
std::shared_ptr<MeshImpl> create_block_impl(DType dt, int64_t nx, int64_t ny, int64_t nzl, const void* x,
                                            const void* y, const void* z, int64_t NX, int64_t NY, int64_t NZ,
                                            int64_t i0, int64_t j0, int64_t k0, int ghost, int gxy);

// Host-side analysis of a network (no device): what each strategy will do.
struct Model {
  int64_t h2d = 0, d2h = 0, kernels = 0;
  int64_t units = 0;  // footprint in problem-array units (scalar 1, vector 4)
};
Model model(const Dag& dag, dfg_strategy s, bool host_mode);
int64_t staged_units(const Dag& dag, const std::vector<int>& order, bool host_mode);
std::vector<int> greedy_staged_order(const Dag& dag);
int64_t predicted_device_bytes(const Dag& dag, dfg_strategy s, int64_t cells, size_t tsize);
int64_t predicted_pcie_bytes(const Dag& dag, dfg_strategy s, int64_t cells, size_t tsize, bool host_mode);

// DFG_HYBRID: staged execution under a device-memory cap with spill-to-host
// (policy in DESIGN.md section 5b).  Planned on the host
// at compile, replayed by exec_hybrid.
struct HybridEvent {
  enum Kind : int { Upload = 0, Reload, Spill, Discard, Drop, Run, SinkD2H, SinkHost, SinkH2D };
  Kind kind;
  Ref ref;
};
struct HybridPlan {
  std::vector<HybridEvent> ev;
  int64_t high = 0;                  // device high-water, units
  int64_t h2d = 0, d2h = 0;          // transfers (host mode: + 4 mesh arrays)
  int64_t h2d_units = 0, d2h_units = 0;
};
// Throws DFG_E_NOMEM if cap_units is below some filter's working set.
HybridPlan plan_hybrid(const Dag& dag, const std::vector<int>& order, int64_t cap_units, bool host);

struct PlanImpl {
  std::shared_ptr<MeshImpl> mesh;
  Dag dag;
  dfg_strategy strategy = DFG_FUSED;
  size_t cap = 0;
  FusedSource fsrc;
  LoadedModule mod;
  int regs = 0, spill = 0;
  int last_variant = 0;  // 1 TMA, 2 general, 3 pointwise, 4 TMA multi-block (dfg_execute_blocks), 5 tile (cp.async ring), 6 tile multi-block,
                         // 7 rows (bulk row copies), 8 rows multi-block
  size_t rows_smem = 0;  // dynamic smem of the row-class kernel (0: unavailable)
  // encoded tensor maps of the last launch (TMA / row-class kernel), reused
  // while the field pointers and the slab view are the same (a time step, a
  // block executed again): cuTensorMapEncodeTiled is host work per map
  struct MapCache {
    std::vector<const void*> ptrs;
    int64_t key[4] = {-1, -1, -1, -1};
    std::vector<unsigned char> maps;
    bool hit(const std::vector<const void*>& f, const int64_t (&k)[4]) const {
      return f == ptrs && std::equal(k, k + 4, key) && !maps.empty();
    }
  };
  MapCache tma_maps, rows_maps;
  uint32_t peer_wait_epoch = 0;  // != 0: the next peer launch waits in the kernel for this step's ready flags
  int64_t last_kz = 0;   // z-chunk length of the last TMA launch
  int last_halo = 0;     // halo of the last execute: 0 none, 1 NCCL, 2 local copies, 3 peer (in place), 4 peer copies
  dfg_stats st{};
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  bool timed = false;
  // dfg_plan_set_timing: 0 no events, 1 execute interval (ev0/ev1), 2 also
  // one event pair per fused-kernel launch.  A timestamped event costs GPU
  // time of its own (~2 us each, measured), which small meshes notice.
  int timing = 1;
  // fused-kernel launch timing: event pairs resolved lazily in stats()
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> kev_free, kev_pending;
  std::pair<cudaEvent_t, cudaEvent_t> kernel_events();
  // bracket one fused launch with a kernel event pair when timing >= 2
  std::pair<cudaEvent_t, cudaEvent_t> kernel_begin(cudaStream_t s);
  void kernel_end(const std::pair<cudaEvent_t, cudaEvent_t>& e, cudaStream_t s);
  void resolve_kernel_times();
  std::map<std::string, std::vector<char>> const_cache;  // roundtrip host constants
  std::vector<int> order;  // staged execution order (list order unless a cap forced a reorder)
  HybridPlan hyb;          // DFG_HYBRID schedule for hyb_host (0 device, 1 host binding mode)
  int hyb_host = -1;
  void plan_hybrid_for(bool host);
  // streamed strategy: ring of chunk slabs and the two copy streams
  std::vector<void*> stream_in, stream_out;
  int64_t stream_C = 0;
  int stream_R = 0;
  bool stream_ready = false;
  cudaStream_t sH2D = nullptr, sD2H = nullptr;
  // multi-slab fused execute: halo exchange on its own stream, overlapped
  // with the interior planes
  cudaStream_t sHalo = nullptr;
  cudaEvent_t evHaloIn = nullptr, evHaloOut = nullptr;
  // staged strategy, everything device-resident: the execute's launches,
  // stream-ordered allocations and frees captured once into a CUDA graph and
  // replayed while the output and input pointers stay the same (DFG_GRAPH=0:
  // off).  gdelta = the counters one execute adds.
  cudaGraphExec_t gexec = nullptr;
  std::vector<const void*> gkey;
  cudaStream_t sCap = nullptr;
  dfg_stats gdelta{};
  int64_t graph_launches = 0;   // executes served by a replay
  ~PlanImpl();
  void execute(void* out, bool out_dev, cudaStream_t s);

 private:
  // kb / ke: global plane range of this launch (default: all owned planes of v)
  // peer: read the planes outside the slab from the linked neighbours' buffers
  // (TMA kernel only; the caller checks tma_peer_ok)
  void launch_fused(const std::vector<const void*>& fptr, void* dout, const void* const tab[3], const SlabView& v,
                    cudaStream_t s, int64_t kb = -1, int64_t ke = -1, bool peer = false);
  bool tma_ok(const std::vector<const void*>& fptr, const void* dout, const SlabView& v) const;
 public:
  // the row-copy kernel's preconditions: 16-byte aligned field bases and
  // plane strides (DFG_FUSED_KERNEL=tile / general turn it off)
  bool rows_ok(const std::vector<const void*>& fptr, const SlabView& v);
 private:
  void exec_fused_peer(const std::vector<const void*>& fptr, void* out, bool out_dev, cudaStream_t s);
  void exec_streamed(void* out, bool out_dev, cudaStream_t s);
  void release_stream_buffers();
  void exec_fused(void* out, bool out_dev, cudaStream_t s);
  void exec_staged(void* out, bool out_dev, cudaStream_t s);
  void exec_staged_graph(void* out, cudaStream_t s);
  void exec_hybrid(void* out, bool out_dev, cudaStream_t s);
  void exec_roundtrip(void* out, bool out_dev, cudaStream_t s);
  void halo_exchange(const std::vector<int>& inputs, cudaStream_t s);
};

// Fused plans of one network on several meshes (VisIt blocks of a device) in
// one launch when they share the generated module and the TMA layout; else
// one execute per plan.  Outputs are device pointers.
void execute_blocks(const std::vector<PlanImpl*>& plans, const std::vector<void*>& outs, cudaStream_t s);

std::unique_ptr<PlanImpl> compile_plan(std::shared_ptr<MeshImpl> mesh, const std::string& expr, dfg_strategy s,
                                       size_t cap);

// NCCL (loaded with dlopen)
void nccl_unique_id(void* out128);
void mesh_init_comm(MeshImpl& m, const void* id128, int rank, int nranks);

// Peer-memory halo: export blob of a z-slab (IPC handles of its bound device
// fields and of its step flags) and the link to the neighbours' blobs.
constexpr size_t kPeerBlobBytes = 4096;
void mesh_peer_export(MeshImpl& m, void* blob);
void mesh_link_peers(MeshImpl& m, const void* lo_blob, const void* hi_blob);
// One TMA read of an exported slab's probe block on the current device;
// true when it returns the pattern (dfg_peer_probe).
bool peer_probe(const void* blob);
// flag word offsets (uint32 units, 64 bytes apart)
constexpr int kFlagReady = 0, kFlagLoDone = 16, kFlagHiDone = 32;

}  // namespace dfg
