// Program tables of the synthetic workloads ("virtual SASS"), docs/EVENT_MODEL.md §3.1-3.4.
// {opcode, kind, width, bb, is_leader, guarded}. Used at compile time by the kernels' hooks and
// exported by nvbt_program(). Basic blocks follow P:L115-117 (§4) (reading R-14).
#pragma once
#include "nvbt.h"

namespace nvbt {
namespace op {
enum : uint16_t { S2R = 0, IMAD, ISETP, EXIT, IMAD_WIDE, LDG, STG, FADD, FFMA, MOV, IADD, BRA, SEL,
                  // §3.6 (F4)
                  SHFL, FMUL, LOP3, I2F, MUFU_SIN, MUFU_COS, FSEL, BREV, SHF, WFFT32 };
}
constexpr uint32_t kWorkloadOpcodes = 16;
constexpr uint32_t kWfftOpcodes = 32;
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
// §3.6 (F4): the kernel that uses the proxy instruction WFFT32 (Listing 10 analogue)
struct ProgWfftEmu {
  static constexpr bool kStageTrace = false;   // k_wfft's own shared memory leaves no room for trace staging
  static constexpr int N = 14;
  static constexpr int REG_LO = 5, REG_HI = 12;
  static constexpr nvbt_instr_desc t[N] = {
      NVBT_D(S2R, ALU, 0, 0, 1, 0),       NVBT_D(S2R, ALU, 0, 0, 0, 0),  NVBT_D(IMAD, ALU, 0, 0, 0, 0),
      NVBT_D(ISETP, ALU, 0, 0, 0, 0),     NVBT_D(EXIT, CTRL, 0, 0, 0, 1),
      NVBT_D(IMAD_WIDE, ALU, 0, 1, 1, 0), NVBT_D(LDG, GLD, 8, 1, 0, 0),  NVBT_D(WFFT32, ALU, 0, 1, 0, 0),
      NVBT_D(IMAD_WIDE, ALU, 0, 1, 0, 0), NVBT_D(STG, GST, 8, 1, 0, 0),  NVBT_D(IADD, ALU, 0, 1, 0, 0),
      NVBT_D(ISETP, ALU, 0, 1, 0, 0),     NVBT_D(BRA, CTRL, 0, 1, 0, 1),
      NVBT_D(EXIT, CTRL, 0, 2, 1, 0)};
};

// §3.6 (F4): the same transform written in CUDA (radix-2 DIF over shuffles)
#define NVBT_TW(b, l) NVBT_D(LOP3, ALU, 0, b, l, 0), NVBT_D(LOP3, ALU, 0, b, 0, 0), NVBT_D(ISETP, ALU, 0, b, 0, 0), \
    NVBT_D(I2F, ALU, 0, b, 0, 0), NVBT_D(MUFU_SIN, ALU, 0, b, 0, 0), NVBT_D(MUFU_COS, ALU, 0, b, 0, 0),            \
    NVBT_D(FSEL, ALU, 0, b, 0, 0), NVBT_D(FSEL, ALU, 0, b, 0, 0)
#define NVBT_ST(b) NVBT_D(SHFL, ALU, 0, b, 0, 0), NVBT_D(SHFL, ALU, 0, b, 0, 0), NVBT_D(FFMA, ALU, 0, b, 0, 0), \
    NVBT_D(FFMA, ALU, 0, b, 0, 0), NVBT_D(FMUL, ALU, 0, b, 0, 0), NVBT_D(FFMA, ALU, 0, b, 0, 0),              \
    NVBT_D(FMUL, ALU, 0, b, 0, 0), NVBT_D(FFMA, ALU, 0, b, 0, 0)
struct ProgWfftSw {
  static constexpr bool kStageTrace = false;   // k_wfft's own shared memory leaves no room for trace staging
  static constexpr int N = 83;
  static constexpr int REG_LO = 39, REG_HI = 81;
  static constexpr nvbt_instr_desc t[N] = {
      NVBT_D(S2R, ALU, 0, 0, 1, 0), NVBT_D(S2R, ALU, 0, 0, 0, 0), NVBT_D(IMAD, ALU, 0, 0, 0, 0),
      NVBT_D(ISETP, ALU, 0, 0, 0, 0), NVBT_D(EXIT, CTRL, 0, 0, 0, 1),
      NVBT_TW(1, 1), NVBT_TW(1, 0), NVBT_TW(1, 0), NVBT_TW(1, 0),
      NVBT_D(BREV, ALU, 0, 1, 0, 0), NVBT_D(SHF, ALU, 0, 1, 0, 0),
      NVBT_D(IMAD_WIDE, ALU, 0, 2, 1, 0), NVBT_D(LDG, GLD, 8, 2, 0, 0),
      NVBT_ST(2), NVBT_ST(2), NVBT_ST(2), NVBT_ST(2),
      NVBT_D(SHFL, ALU, 0, 2, 0, 0), NVBT_D(SHFL, ALU, 0, 2, 0, 0), NVBT_D(FFMA, ALU, 0, 2, 0, 0),
      NVBT_D(FFMA, ALU, 0, 2, 0, 0),
      NVBT_D(IMAD_WIDE, ALU, 0, 2, 0, 0), NVBT_D(STG, GST, 8, 2, 0, 0), NVBT_D(IADD, ALU, 0, 2, 0, 0),
      NVBT_D(ISETP, ALU, 0, 2, 0, 0), NVBT_D(BRA, CTRL, 0, 2, 0, 1),
      NVBT_D(EXIT, CTRL, 0, 3, 1, 0)};
};
#undef NVBT_TW
#undef NVBT_ST
#undef NVBT_D

}  // namespace nvbt
