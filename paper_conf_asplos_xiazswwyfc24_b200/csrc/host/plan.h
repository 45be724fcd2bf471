// A lowered plan: analysis results + per-subprogram stage lists + workspace layout + bindings.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../exec_types.h"
#include "bert.h"
#include "lstm.h"
#include "mmoe.h"
#include "swin.h"
#include "se.h"
#include "mbconv.h"
#include "resnext.h"
#include "ir.h"

namespace souffle {

// TMA descriptor request (encoded at souffle_workspace_init, when pointers are known)
struct TmapSpec {
  int32_t buf;        // bound buffer index, or -1 for workspace
  int64_t byte_off;   // byte offset inside the buffer / workspace data region
  int64_t rows, cols; // 2-D bf16 tensor [rows, cols], row stride = cols elements
  int32_t box_rows;   // box = {64 cols, box_rows rows}, 128B swizzle
};

// workspace layout (bytes from the workspace base pointer)
struct WsLayout {
  int64_t ctrl_off = 0, ctrl_bytes = 256;
  int64_t prog_off = 0, prog_bytes = 0;   // stages|members|ins|addrs|tabs|tmaps|zero list
  int64_t data_off = 0, data_bytes = 0;   // intermediates and accumulators
  int64_t total = 0;
  // sub-offsets inside the program region
  int64_t o_stages = 0, o_members = 0, o_ins = 0, o_addrs = 0, o_tabs = 0, o_tmaps = 0, o_zero = 0;
};

struct Plan {
  Graph g;                 // copy of the user graph (plan independent of it afterwards)
  Analysis an;
  souffle_device_desc dev{};
  uint32_t flags = 0;

  // lowered program
  std::vector<Stage> stages;
  std::vector<GemmMember> members;
  std::vector<Ins> ins;
  std::vector<Addr> addrs;
  std::vector<int32_t> tabs;
  std::vector<TmapSpec> tmaps;
  std::vector<Launch> launches;
  std::vector<int64_t> zero_list;  // (byte offset in data region, bytes) pairs
  WsLayout ws;
  int32_t n_barriers = 0;
  std::string text;                 // describe()

  // bindings: placeholder/output node -> buffer slot
  std::vector<int32_t> node_buf;    // -1 if not bindable
  std::vector<void*> buf_ptr;       // per slot
  std::vector<int32_t> buf_node;    // slot -> node
  void* inited_ws = nullptr;        // workspace the program/tmaps were uploaded to
  bool dirty = true;
  bool profiling = false;
  std::vector<uint8_t> host_prog;   // packed program region (uploaded by workspace_init)
  BertPlan bert;                    // pattern lowering (bert.on: kernels/bert.cu runs the program)
  LstmPlan lstm;                    // pattern lowering (lstm.on: kernels/lstm.cu runs the program)
  MmoePlan mmoe;                    // pattern lowering (mmoe.on: kernels/mmoe.cu runs the program)
  SwinPlan swin;                    // pattern lowering (swin.on: kernels/swin.cu, one CUDA graph)
  SePlan se;                        // pattern lowering (se.on: kernels/se.cu, EfficientNet M0-M9)
  MbPlan mb;                        // pattern lowering (mb.on: kernels/mbconv.cu, MBConv blocks M0-M9)
  RxPlan rx;                        // pattern lowering (rx.on: kernels/resnext.cu, ResNeXt blocks R0-R7)
  ~Plan();
};

void lower(Plan& p);              // fills the lowered program + layout (pure host)
void pack_program(Plan& p, const std::vector<uint8_t>* tmap_bytes);

}  // namespace souffle
