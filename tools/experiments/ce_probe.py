"""Does a small H2D copy on one stream wait behind a large H2D copy on another?"""
import torch

side = torch.cuda.Stream()
big_h = torch.empty(16 << 20, dtype=torch.uint8).pin_memory()
big_d = torch.empty(16 << 20, dtype=torch.uint8, device="cuda")
small_h = torch.empty(80_000, dtype=torch.uint8).pin_memory()
small_d = torch.empty(80_000, dtype=torch.uint8, device="cuda")
for _ in range(3):
    big_d.copy_(big_h, non_blocking=True)
    small_d.copy_(small_h, non_blocking=True)
torch.cuda.synchronize()
for trial in range(3):
    e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    torch.cuda.synchronize()
    e[0].record(side)
    with torch.cuda.stream(side):
        big_d.copy_(big_h, non_blocking=True)
    e[1].record(side)
    torch.cuda._sleep(20_000)  # ~10 us so the big copy is underway
    e[2].record()
    small_d.copy_(small_h, non_blocking=True)
    e[3].record()
    torch.cuda.synchronize()
    print(f"big {e[0].elapsed_time(e[1])*1e3:.0f} us; small issued at {e[0].elapsed_time(e[2])*1e3:.0f} us "
          f"took {e[2].elapsed_time(e[3])*1e3:.0f} us")
print("asyncEngineCount", torch.cuda.get_device_properties(0))
