// spp_format.h — product-side constants of FORMAT.md v1 (host encoders and
// CUDA decoders of libspp).  Independent of oracle/ (which re-implements
// FORMAT.md on its own).
#pragma once
#include <stdint.h>

namespace spp {

constexpr uint32_t kCosmoMagic = 0x43505053u;    // "SPPC"
constexpr uint32_t kDeepcamMagic = 0x44505053u;  // "SPPD"
constexpr uint16_t kVersion = 1;
constexpr int kHeaderBytes = 64;

// CosmoFlow header field offsets (FORMAT.md 1.1)
namespace cosmo {
constexpr int kC = 8, kD = 10, kH = 12, kW = 14, kNU = 16, kNSlab = 20, kUOff = 24, kSlabOff = 32,
              kTotal = 40;
constexpr int kSlabBytes = 32;                   // {z0, z1, G, kw, pad[3], lut_off, keys_off}
constexpr int kMaxU = 32768;
constexpr int kMaxG2 = 65536;                    // 16-bit keys
constexpr int kMaxG1 = 256;                      // 8-bit keys
constexpr int kRawSlab = 8;                      // RAW escape key width
constexpr int kEscaped = 3;                      // escaped 1-byte keys (FORMAT.md 1.5)
constexpr int kEscBlock = 256;                   // voxels per eidx entry
}  // namespace cosmo

// DeepCAM header field offsets (FORMAT.md 2.1)
namespace deepcam {
constexpr int kC = 8, kH = 10, kW = 12, kAlign = 14, kL = 16, kDirOff = 24, kPayloadOff = 32, kTotal = 40;
constexpr uint8_t kModeRaw = 0, kModeSeg = 1, kModeRaw16 = 2, kModeSegRaw = 3;  // 2.6 RAW16, 2.7 SEG+RAW
constexpr uint8_t kRepeat = 0, kDiff = 1, kRawSeg = 2;  // kRawSeg: FORMAT.md 2.7
constexpr int kEminBias = 150;                   // emin = emin_b - 150
constexpr int kEminBMin = 1, kEminBMax = 246;    // emin in [-149, 96]
constexpr int kRepeatMin = 16;                   // encoder: identical run that opens a REPEAT
constexpr int kLookahead = 64;                   // encoder: emin lookahead window
constexpr int kMaxCode = 1984;                   // largest code magnitude (31 << 6)
constexpr int64_t kMaxAbsS = 1983LL * 1984LL;    // encoder bound on |S|
}  // namespace deepcam

inline uint64_t round_up16(uint64_t x) { return (x + 15) & ~uint64_t(15); }

}  // namespace spp
