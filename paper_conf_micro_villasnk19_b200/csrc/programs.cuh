// Program tables of the synthetic workloads ("virtual SASS"), docs/EVENT_MODEL.md §3.1-3.4.
// {opcode, kind, width, bb, is_leader, guarded}. Used at compile time by the kernels' hooks and
// exported by nvbt_program(). Basic blocks follow P:L115-117 (§4) (reading R-14).
#pragma once
#include "nvbt.h"

namespace nvbt {
namespace op {
enum : uint16_t { S2R = 0, IMAD, ISETP, EXIT, IMAD_WIDE, LDG, STG, FADD, FFMA, MOV, IADD, BRA, SEL };
}
constexpr uint32_t kWorkloadOpcodes = 16;
constexpr uint8_t ALU = NVBT_K_ALU, CTRL = NVBT_K_CTRL, GLD = NVBT_K_GLD, GST = NVBT_K_GST;

#define NVBT_D(o, k, w, b, l, g) nvbt_instr_desc{op::o, k, w, b, l, g, 0}

// REG_LO..REG_HI: pcs inside loops; their hooks accumulate in registers (flushed once per warp). Other
// hooks run once per warp and add straight into the CTA's shared bins.
struct ProgVectorAdd {  // §3.1
  static constexpr int N = 13;
  static constexpr int REG_LO = 1, REG_HI = 0;
  static constexpr nvbt_instr_desc t[N] = {
      NVBT_D(S2R, ALU, 0, 0, 1, 0),       NVBT_D(S2R, ALU, 0, 0, 0, 0),       NVBT_D(IMAD, ALU, 0, 0, 0, 0),
      NVBT_D(ISETP, ALU, 0, 0, 0, 0),     NVBT_D(EXIT, CTRL, 0, 0, 0, 1),     NVBT_D(IMAD_WIDE, ALU, 0, 1, 1, 0),
      NVBT_D(IMAD_WIDE, ALU, 0, 1, 0, 0), NVBT_D(LDG, GLD, 4, 1, 0, 0),       NVBT_D(LDG, GLD, 4, 1, 0, 0),
      NVBT_D(IMAD_WIDE, ALU, 0, 1, 0, 0), NVBT_D(FADD, ALU, 0, 1, 0, 0),      NVBT_D(STG, GST, 4, 1, 0, 0),
      NVBT_D(EXIT, CTRL, 0, 1, 0, 0)};
};

struct ProgSgemm {  // §3.2
  static constexpr int N = 18;
  static constexpr int REG_LO = 10, REG_HI = 15;
  static constexpr nvbt_instr_desc t[N] = {
      NVBT_D(S2R, ALU, 0, 0, 1, 0),  NVBT_D(S2R, ALU, 0, 0, 0, 0),   NVBT_D(S2R, ALU, 0, 0, 0, 0),
      NVBT_D(S2R, ALU, 0, 0, 0, 0),  NVBT_D(IMAD, ALU, 0, 0, 0, 0),  NVBT_D(IMAD, ALU, 0, 0, 0, 0),
      NVBT_D(ISETP, ALU, 0, 0, 0, 0), NVBT_D(EXIT, CTRL, 0, 0, 0, 1), NVBT_D(MOV, ALU, 0, 1, 1, 0),
      NVBT_D(MOV, ALU, 0, 1, 0, 0),  NVBT_D(LDG, GLD, 4, 2, 1, 0),   NVBT_D(LDG, GLD, 4, 2, 0, 0),
      NVBT_D(FFMA, ALU, 0, 2, 0, 0), NVBT_D(IADD, ALU, 0, 2, 0, 0),  NVBT_D(ISETP, ALU, 0, 2, 0, 0),
      NVBT_D(BRA, CTRL, 0, 2, 0, 1), NVBT_D(STG, GST, 4, 3, 1, 0),   NVBT_D(EXIT, CTRL, 0, 3, 0, 0)};
};

struct ProgBfs {  // §3.3 (kernel 1: pcs 0-21, kernel 2: pcs 22-35)
  static constexpr int N = 36;
  static constexpr int REG_LO = 13, REG_HI = 20;
  static constexpr nvbt_instr_desc t[N] = {
      NVBT_D(S2R, ALU, 0, 0, 1, 0),   NVBT_D(S2R, ALU, 0, 0, 0, 0),   NVBT_D(IMAD, ALU, 0, 0, 0, 0),
      NVBT_D(ISETP, ALU, 0, 0, 0, 0), NVBT_D(EXIT, CTRL, 0, 0, 0, 1),
      NVBT_D(LDG, GLD, 1, 1, 1, 0),   NVBT_D(ISETP, ALU, 0, 1, 0, 0), NVBT_D(BRA, CTRL, 0, 1, 0, 1),
      NVBT_D(STG, GST, 1, 2, 1, 0),   NVBT_D(LDG, GLD, 4, 2, 0, 0),   NVBT_D(LDG, GLD, 4, 2, 0, 0),
      NVBT_D(ISETP, ALU, 0, 2, 0, 0), NVBT_D(BRA, CTRL, 0, 2, 0, 1),
      NVBT_D(LDG, GLD, 4, 3, 1, 0),   NVBT_D(LDG, GLD, 1, 3, 0, 0),   NVBT_D(ISETP, ALU, 0, 3, 0, 0),
      NVBT_D(BRA, CTRL, 0, 3, 0, 1),
      NVBT_D(STG, GST, 1, 4, 1, 0),
      NVBT_D(IADD, ALU, 0, 5, 1, 0),  NVBT_D(ISETP, ALU, 0, 5, 0, 0), NVBT_D(BRA, CTRL, 0, 5, 0, 1),
      NVBT_D(EXIT, CTRL, 0, 6, 1, 0),
      NVBT_D(S2R, ALU, 0, 7, 1, 0),   NVBT_D(S2R, ALU, 0, 7, 0, 0),   NVBT_D(IMAD, ALU, 0, 7, 0, 0),
      NVBT_D(ISETP, ALU, 0, 7, 0, 0), NVBT_D(EXIT, CTRL, 0, 7, 0, 1),
      NVBT_D(LDG, GLD, 1, 8, 1, 0),   NVBT_D(ISETP, ALU, 0, 8, 0, 0), NVBT_D(BRA, CTRL, 0, 8, 0, 1),
      NVBT_D(STG, GST, 1, 9, 1, 0),   NVBT_D(STG, GST, 1, 9, 0, 0),   NVBT_D(STG, GST, 4, 9, 0, 0),
      NVBT_D(STG, GST, 1, 9, 0, 0),   NVBT_D(STG, GST, 4, 9, 0, 0),
      NVBT_D(EXIT, CTRL, 0, 10, 1, 0)};
};

struct ProgStencil {  // §3.4
  static constexpr int N = 21;
  static constexpr int REG_LO = 1, REG_HI = 0;
  static constexpr nvbt_instr_desc t[N] = {
      NVBT_D(S2R, ALU, 0, 0, 1, 0),   NVBT_D(S2R, ALU, 0, 0, 0, 0),   NVBT_D(S2R, ALU, 0, 0, 0, 0),
      NVBT_D(S2R, ALU, 0, 0, 0, 0),   NVBT_D(IMAD, ALU, 0, 0, 0, 0),  NVBT_D(IMAD, ALU, 0, 0, 0, 0),
      NVBT_D(ISETP, ALU, 0, 0, 0, 0), NVBT_D(EXIT, CTRL, 0, 0, 0, 1),
      NVBT_D(ISETP, ALU, 0, 1, 1, 0), NVBT_D(LDG, GLD, 4, 1, 0, 0),
      NVBT_D(LDG, GLD, 4, 1, 0, 1),   NVBT_D(LDG, GLD, 4, 1, 0, 1),   NVBT_D(LDG, GLD, 4, 1, 0, 1),
      NVBT_D(LDG, GLD, 4, 1, 0, 1),   NVBT_D(FADD, ALU, 0, 1, 0, 1),  NVBT_D(FADD, ALU, 0, 1, 0, 1),
      NVBT_D(FADD, ALU, 0, 1, 0, 1),  NVBT_D(FFMA, ALU, 0, 1, 0, 1),  NVBT_D(SEL, ALU, 0, 1, 0, 0),
      NVBT_D(STG, GST, 4, 1, 0, 0),   NVBT_D(EXIT, CTRL, 0, 1, 0, 0)};
};
#undef NVBT_D

}  // namespace nvbt
